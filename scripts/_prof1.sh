set -x
mkdir -p gpurun_out/p1
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm --format=csv > gpurun_out/p1/clk.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_star_query -c 4 -o gpurun_out/p1/star python scripts/profile_ssb.py 20 3.1,2.1,1.1,4.3 > gpurun_out/p1/ncu.log 2>&1
for i in 0 1 2 3; do python scripts/src_hot.py gpurun_out/p1/star.ncu-rep 40 $i > gpurun_out/p1/src_hot_$i.txt 2>&1; done
ncu -i gpurun_out/p1/star.ncu-rep --page details > gpurun_out/p1/star.details.txt 2>&1
ncu -i gpurun_out/p1/star.ncu-rep --page raw --csv > gpurun_out/p1/star.raw.csv 2>&1
rm -f gpurun_out/p1/star.ncu-rep
