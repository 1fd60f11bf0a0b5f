set -x
R=gpurun_out/ab6
mkdir -p $R
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_star_query.py -m gpu -q -x > $R/tests.log 2>&1; echo "tests rc=$?"
timeout 1500 python scripts/tile_sweep.py --ab $R/ab.json dfor_d1,dfor_near,dfor_sorted,dfor_consec,for_b16 build_ab/libtilepack_r1.so build_ab/libtilepack_v25.so build_ab/libtilepack_v27.so > $R/ab.log 2>&1
timeout 1200 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v25.so build_ab/libtilepack_v27.so > $R/ssb.log 2>&1
