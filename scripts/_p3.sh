R=gpurun_out/p3
mkdir -p $R
for lib in r1 v10; do
for c in rfor_runs8 rfor_runs64; do
  f=$R/${c}_${lib}
  TILEPACK_LIB_OVERRIDE=$PWD/build_ab/libtilepack_$lib.so timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_decode -s 2 -c 1 -o $f python scripts/profile_one.py "$c" sum 200000000 > $f.log 2>&1
  python scripts/src_hot.py $f.ncu-rep 30 > $f.src.txt 2>&1
  ncu -i $f.ncu-rep --page raw --csv > $f.raw.csv 2>&1
  rm -f $f.ncu-rep
done
done
