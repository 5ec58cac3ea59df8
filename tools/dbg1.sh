O=gpurun_out/dbg1; mkdir -p $O
timeout 900 python bench.py > $O/b_c2.log 2>&1; echo "c2 rc=$?"; tail -1 $O/b_c2.log | cut -c1-1500
GUM_BENCH_DEVICE=0 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --config C1 --steps 3 --warmup 3 > $O/b_mp.log 2>&1; echo "mp rc=$?"; grep metric $O/b_mp.log | tail -1 | cut -c1-2500
timeout 900 python bench.py --config C1 --alg dpr --steps 5 --warmup 3 > $O/b_dpr.log 2>&1; echo "dpr rc=$?"; tail -1 $O/b_dpr.log | cut -c1-1200
