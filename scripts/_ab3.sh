R=gpurun_out/ab3
mkdir -p $R
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v7.so 16 2 > $R/dec16a.log 2>&1
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_v8.so build_ab/libtilepack_v6.so 16 2 > $R/dec16b.log 2>&1
