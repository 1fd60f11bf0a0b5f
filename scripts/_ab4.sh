R=gpurun_out/ab4
mkdir -p $R
timeout 2400 python scripts/tile_sweep.py --ab $R/ab_dfor.json dfor_d1,dfor_near,dfor_sorted,dfor_consec,rfor_runs4,for_b4 build_ab/libtilepack_r1.so build_ab/libtilepack_v14.so build_ab/libtilepack_v18.so > $R/ab.log 2>&1
