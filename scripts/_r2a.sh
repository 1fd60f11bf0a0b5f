set -x
R=gpurun_out/r2a
mkdir -p $R
nvidia-smi -q -d CLOCK > $R/clocks.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x > $R/gpu_tests.log 2>&1; echo "tests rc=$?"
timeout 900 python bench.py > $R/bench.log 2>&1; echo "bench rc=$?"
timeout 300 python bench.py --impl reference --steps 5 --warmup 1 > $R/bench_ref.log 2>&1; echo "ref rc=$?"
timeout 1500 bash scripts/issue_profile.sh > $R/issue.log 2>&1; echo "issue rc=$?"
cp profiles/r02_issue.json $R/ 2>/dev/null
