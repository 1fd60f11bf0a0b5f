set -x
R=gpurun_out/ab2
mkdir -p $R
timeout 900 python -m pytest tests/test_star_query.py tests/test_device_api.py -m gpu -q -x > $R/tests.log 2>&1; echo "tests rc=$?"
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v6.so > $R/ssb.log 2>&1
timeout 400 python scripts/ab_decode.py build_ab/libtilepack_r1.so build_ab/libtilepack_v6.so 16 2 > $R/dec16.log 2>&1
for c in rfor_runs4:global dfor_d1_2^28:sum rfor_runs4:sum; do
  n=${c%%:*}; m=${c##*:}; f=$R/${n//^/}_$m
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_decode -s 2 -c 1 -o $f python scripts/profile_one.py "$n" $m > $f.log 2>&1
  python scripts/src_hot.py $f.ncu-rep 45 > $f.src.txt 2>&1
  ncu -i $f.ncu-rep --page details > $f.details.txt 2>&1
  rm -f $f.ncu-rep
done
