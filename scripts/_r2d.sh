set -x
R=gpurun_out/r2d
mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q -x > $R/gpu_tests.log 2>&1; echo "tests rc=$?"
timeout 600 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v10.so build_ab/libtilepack_v12.so 16 2 > $R/dec16.log 2>&1
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v10.so build_ab/libtilepack_v11.so > $R/ssb.log 2>&1
timeout 900 python scripts/bench_suite.py --reps 5 --out $R/suite.json > $R/suite.log 2>&1
