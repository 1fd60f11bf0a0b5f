set -x
mkdir -p gpurun_out/r
nvidia-smi -q -d CLOCK > gpurun_out/r/clocks.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/r/gpu_tests.log 2>&1; echo "tests rc=$?"
timeout 300 python bench.py > gpurun_out/r/bench.log 2>&1; echo "bench rc=$?"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r/launches_bench.csv python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 2 > /dev/null 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:k_decode_sum -s 3 -c 1 -o gpurun_out/r/bench_full python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > /dev/null 2>&1
python scripts/ncu_summarize.py gpurun_out/r/bench_full.ncu-rep for_b16_sum --algorithmic-bytes 1046875016 > gpurun_out/r/ncu_sum.log 2>&1
cp profiles/ncu_summary.json gpurun_out/r/ncu_summary.json
ncu -i gpurun_out/r/bench_full.ncu-rep --page details > gpurun_out/r/bench_full.details.txt 2>&1; rm -f gpurun_out/r/bench_full.ncu-rep
timeout 900 python scripts/bench_suite.py --reps 5 --out gpurun_out/r/suite.json > gpurun_out/r/suite.log 2>&1; echo "suite rc=$?"
timeout 600 python scripts/bench_ssb.py --sf 20 --check --out gpurun_out/r/ssb_sf20.json > gpurun_out/r/ssb.log 2>&1; echo "ssb rc=$?"
timeout 400 python scripts/bench_ssb.py --sf 20 --scheme none --out gpurun_out/r/ssb_sf20_none.json > gpurun_out/r/ssb_none.log 2>&1; echo "ssb none rc=$?"
timeout 600 python scripts/bench_encode.py --out gpurun_out/r/encode.json > gpurun_out/r/encode.log 2>&1; echo "enc rc=$?"
