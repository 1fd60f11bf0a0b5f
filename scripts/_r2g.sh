set -x
R=gpurun_out/r2g
mkdir -p $R
timeout 900 python -m pytest tests/test_star_query.py tests/test_ssb.py -m gpu -q -x > $R/tests.log 2>&1; echo "tests rc=$?"
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_v14.so build_ab/libtilepack_v18.so build_ab/libtilepack_v19.so > $R/ssb.log 2>&1
timeout 600 python scripts/bench_suite.py --reps 5 --only dfor --out $R/suite_dfor.json > $R/suite_dfor.log 2>&1
