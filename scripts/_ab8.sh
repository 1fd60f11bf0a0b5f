R=gpurun_out/ab8
mkdir -p $R
timeout 1500 python scripts/tile_sweep.py --ab $R/ab.json rfor_runs4,rfor_runs8,dfor_d1,dfor_near,for_b4,for_b16 build_ab/libtilepack_v31.so build_ab/libtilepack_v32.so build_ab/libtilepack_v33.so > $R/ab.log 2>&1
