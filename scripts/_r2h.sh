set -x
R=gpurun_out/r2h
mkdir -p $R
timeout 900 python bench.py --steps 20 --warmup 5 > $R/bench.log 2>&1; echo "bench rc=$?"
TILEPACK_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 5 --warmup 3 > $R/bench_2rank_gloo.log 2>&1; echo "2rank rc=$?"
timeout 900 python scripts/ab_ssb.py build_ab/libtilepack_r1.so build_ab/libtilepack_v31.so > $R/ssb.log 2>&1
