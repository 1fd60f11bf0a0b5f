set -x
R=gpurun_out/p2
mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_star_query -c 3 -o $R/star python scripts/profile_ssb.py 20 3.1,1.1,2.1 > $R/ncu.log 2>&1
for i in 0 1 2; do python scripts/src_hot.py $R/star.ncu-rep 45 $i > $R/src_hot_$i.txt 2>&1; done
ncu -i $R/star.ncu-rep --page details > $R/star.details.txt 2>&1
ncu -i $R/star.ncu-rep --page raw --csv > $R/star.raw.csv 2>&1
rm -f $R/star.ncu-rep
