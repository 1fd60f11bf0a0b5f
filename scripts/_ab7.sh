set -x
R=gpurun_out/ab7
mkdir -p $R
timeout 1500 python -m pytest tests -m gpu -q > $R/tests.log 2>&1; echo "tests rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $R/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python scripts/tile_sweep.py --ab $R/ab.json for_b1,for_b4,for_b8,for_b12,for_b16 build_ab/libtilepack_r1.so build_ab/libtilepack_v29.so build_ab/libtilepack_v28.so > $R/ab.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --no-schemes --no-ssb --no-cpu-baseline > $R/bench.log 2>&1
