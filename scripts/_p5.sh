R=gpurun_out/p5
mkdir -p $R
TILEPACK_LIB_OVERRIDE=$PWD/build_ab/libtilepack_prof.so timeout 600 python scripts/prof_waits.py 20 1.1,1.2,1.3,2.1,2.2,2.3,3.1,3.2,3.3,3.4,4.1,4.2,4.3 > $R/waits.log 2>&1
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_v14.so build_ab/libtilepack_v17.so > $R/ssb.log 2>&1
