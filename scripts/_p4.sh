R=gpurun_out/p4
mkdir -p $R
for lib in r1 v13; do
  TILEPACK_LIB_OVERRIDE=$PWD/build_ab/libtilepack_$lib.so timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_star_query -c 2 -o $R/star_$lib python scripts/profile_ssb.py 20 2.1,4.1 > $R/ncu_$lib.log 2>&1
  for i in 0 1; do python scripts/src_hot.py $R/star_$lib.ncu-rep 40 $i > $R/src_${lib}_$i.txt 2>&1; done
  ncu -i $R/star_$lib.ncu-rep --page raw --csv > $R/star_$lib.raw.csv 2>&1
  rm -f $R/star_$lib.ncu-rep
done
timeout 2400 python scripts/tile_sweep.py --run2 $R/tile_sweep2.json > $R/tile_sweep2.log 2>&1
