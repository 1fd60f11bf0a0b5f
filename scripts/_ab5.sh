R=gpurun_out/ab5
mkdir -p $R
timeout 2400 python scripts/tile_sweep.py --ab $R/ab.json for_b4,for_b16,rfor_runs4,dfor_d1 build_ab/libtilepack_r1.so build_ab/libtilepack_v23.so build_ab/libtilepack_v24.so build_ab/libtilepack_v25.so > $R/ab.log 2>&1
timeout 1200 python scripts/ab_ssb.py build_ab/libtilepack_v18.so build_ab/libtilepack_v20.so build_ab/libtilepack_v21.so build_ab/libtilepack_v22.so > $R/ssb.log 2>&1
