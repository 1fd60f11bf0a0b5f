set -x
R=gpurun_out/r2f
mkdir -p $R
timeout 900 python -m pytest tests/test_star_query.py tests/test_ssb.py tests/test_gpu_parity.py -m gpu -q -x > $R/tests.log 2>&1; echo "tests rc=$?"
timeout 600 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v14.so 16 2 > $R/dec16.log 2>&1
timeout 1200 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v14.so build_ab/libtilepack_v15.so build_ab/libtilepack_v16.so > $R/ssb.log 2>&1
