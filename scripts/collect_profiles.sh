#!/bin/bash
# Copy one refresh_profiles.sh run (gpurun_out/<dir>) into profiles/r02_* and regenerate the README.
#   bash scripts/collect_profiles.sh gpurun_out/r2f
set -e
R=${1:-gpurun_out/r2f}
P=profiles
grep '^{' $R/bench.log | tail -1 > $P/r02_bench.json
grep '^{' $R/bench_ref.log | tail -1 > $P/r02_bench_reference.json || true
cp $R/launches_bench.csv $P/r02_launches_bench.csv
cp $R/ncu_summary.json $P/ncu_summary.json
cp $R/bench_full.details.txt $P/r02_ncu_k_decode_sum_details.txt
cp $R/suite.json $P/r02_suite.json
cp $R/r02_issue.json $P/r02_issue.json 2>/dev/null || true
cp $R/ssb_sf20.json $P/r02_ssb_sf20.json
cp $R/ssb_sf20_none.json $P/r02_ssb_sf20_none.json
cp $R/ssb_sf160.json $P/r02_ssb_sf160.json
cp $R/star.details.txt $P/r02_star_details.txt
for i in 0 1 2 3; do cp $R/star_src_hot_$i.txt $P/r02_star_src_hot_q$i.txt; done
cp $R/star_waits.txt $P/r02_star_waits.txt
cp $R/encode.json $P/r02_encode.json
cp $R/random_access.json $P/r02_random_access.json
cp $R/cascaded.json $P/r02_cascaded_ablation.json
cp $R/nomb.json $P/r02_nomb_ablation.json
cp $R/gpu_tests.log $P/r02_gpu_tests.log
cp $R/clocks.txt $P/r02_clocks.txt
python scripts/profiles_readme.py > /dev/null
