set -x
R=gpurun_out/r2e
mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q -x > $R/gpu_tests.log 2>&1; echo "tests rc=$?"
timeout 600 python scripts/bench_suite.py --reps 5 --only dfor --out $R/suite_dfor.json > $R/suite_dfor.log 2>&1
timeout 600 python scripts/bench_suite.py --reps 5 --only rfor --out $R/suite_rfor.json > $R/suite_rfor.log 2>&1
timeout 600 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v13.so 16 2 > $R/dec16.log 2>&1
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v13.so > $R/ssb.log 2>&1
timeout 1500 python scripts/tile_sweep.py --run $R/tile_sweep.json > $R/tile_sweep.log 2>&1
