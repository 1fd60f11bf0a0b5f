set -x
R=gpurun_out/r2b
mkdir -p $R
timeout 900 python -m pytest tests/test_star_query.py tests/test_ssb.py -m gpu -q -x > $R/star_tests.log 2>&1; echo "star tests rc=$?"
timeout 600 python bench.py --steps 20 --no-schemes --no-cpu-baseline > $R/bench.log 2>&1; echo "bench rc=$?"
timeout 300 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_r2.so 16 3 > $R/ab16.log 2>&1
timeout 300 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_r2.so 4 2 > $R/ab4.log 2>&1
timeout 900 python -m pytest tests -m gpu -q > $R/gpu_tests.log 2>&1; echo "all tests rc=$?"
