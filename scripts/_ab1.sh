set -x
R=gpurun_out/ab1
mkdir -p $R
timeout 1200 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v1.so build_ab/libtilepack_v2.so build_ab/libtilepack_v3.so build_ab/libtilepack_v4.so > $R/ssb.log 2>&1
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v1.so 16 2 > $R/dec16.log 2>&1
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_v5.so build_ab/libtilepack_r1.so 16 2 >> $R/dec16.log 2>&1
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_v5.so build_ab/libtilepack_r1.so 4 2 > $R/dec4.log 2>&1
