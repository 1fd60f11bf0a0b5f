#!/bin/bash
# One box, one commit: every measurement under profiles/ (outputs in gpurun_out/r2f/, copied by
# scripts/collect_profiles.sh to profiles/r02_*).   gpurun --timeout 5400 -- 'bash scripts/refresh_profiles.sh'
set -x
R=gpurun_out/r2f
mkdir -p $R
nvidia-smi -q -d CLOCK > $R/clocks.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $R/gpu_tests.log 2>&1; echo "tests rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > $R/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $R/bench.log 2>&1; echo "bench rc=$?"
timeout 300 python bench.py --impl reference --steps 5 --warmup 1 > $R/bench_ref.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file $R/launches_bench.csv python bench.py --steps 10 --warmup 3 --quick --e2e-steps 2 > /dev/null 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:k_decode_sum -s 3 -c 1 -o $R/bench_full python bench.py --steps 3 --warmup 3 --quick --e2e-steps 1 > /dev/null 2>&1
python scripts/ncu_summarize.py $R/bench_full.ncu-rep for_b16_sum --algorithmic-bytes 1046875016 > $R/ncu_sum.log 2>&1
cp profiles/ncu_summary.json $R/ncu_summary.json
ncu -i $R/bench_full.ncu-rep --page details > $R/bench_full.details.txt 2>&1; rm -f $R/bench_full.ncu-rep
timeout 1200 python scripts/bench_suite.py --reps 5 --out $R/suite.json > $R/suite.log 2>&1; echo "suite rc=$?"
timeout 1500 bash scripts/issue_profile.sh > $R/issue.log 2>&1; cp profiles/r02_issue.json $R/ 2>/dev/null
timeout 900 python scripts/bench_ssb.py --sf 20 --check --out $R/ssb_sf20.json > $R/ssb.log 2>&1; echo "ssb rc=$?"
timeout 600 python scripts/bench_ssb.py --sf 20 --scheme none --out $R/ssb_sf20_none.json > $R/ssb_none.log 2>&1; echo "ssb none rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_star_query -c 4 -o $R/star python scripts/profile_ssb.py 20 1.1,2.1,3.1,4.1 > $R/star_ncu.log 2>&1
for i in 0 1 2 3; do python scripts/src_hot.py $R/star.ncu-rep 40 $i > $R/star_src_hot_$i.txt 2>&1; done
ncu -i $R/star.ncu-rep --page details > $R/star.details.txt 2>&1; rm -f $R/star.ncu-rep
python scripts/build_variant.py prof "-DTP_PROFILE_WAITS" > /dev/null 2>&1
TILEPACK_LIB_OVERRIDE=$PWD/build_ab/libtilepack_prof.so timeout 600 python scripts/prof_waits.py 20 1.1,1.2,1.3,2.1,2.2,2.3,3.1,3.2,3.3,3.4,4.1,4.2,4.3 > $R/star_waits.txt 2>&1
timeout 1200 python scripts/bench_ssb.py --sf 160 --reps 5 --out $R/ssb_sf160.json > $R/ssb160.log 2>&1; echo "ssb160 rc=$?"
timeout 900 python scripts/bench_encode.py --out $R/encode.json > $R/encode.log 2>&1; echo "enc rc=$?"
timeout 600 python scripts/bench_random_access.py --reps 5 --out $R/random_access.json > $R/ra.log 2>&1; echo "ra rc=$?"
timeout 600 python scripts/bench_cascaded.py --out $R/cascaded.json > $R/cascaded.log 2>&1; echo "cascaded rc=$?"
timeout 600 python scripts/bench_nomb.py --out $R/nomb.json > $R/nomb.log 2>&1; echo "nomb rc=$?"
