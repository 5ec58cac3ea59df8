#!/bin/bash
# Round-end measurement (1 GPU): GPU suite, smoke, bench lines for every config (+ reference arm), launch lists,
# advance DRAM traffic, ncu --set full of the dominant kernels, ablations. Outputs under gpurun_out/final.
O=gpurun_out/final; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err; echo "ref rc=$?"
for f in C1 C2 C3 C4 C5; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'], (d.get('detail') or {}).get('parity_full_size',{}).get('exact'), d['e2e'] and round(d['e2e']['value'],2))"; done
P="python tools/profile_run.py --runs 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C4_wcc.csv $P --config C4 --alg wcc > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C5_pr.csv $P --config C5 --alg pr > /dev/null 2>&1
for cfg in "C2 bfs degree" "C4 wcc seg" "C5 pr seg"; do set -- $cfg
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_$1_$2.csv $P --config $1 --alg $2 --part $3 > /dev/null 2>&1
done
echo "ncu lists done"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 3 -c 1 -o $O/adv_C2_bfs $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_filter -s 2 -c 1 -o $O/filt_C2_bfs $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 10 -c 1 -o $O/adv_C5_pr $P --config C5 --alg pr > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tail -s 40 -c 1 -o $O/tail_C3_sssp $P --config C3 --alg sssp > /dev/null 2>&1
echo "ncu full done"
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal.txt 2>&1
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --split --out $O/abl_fsteal_split.json > $O/abl_fsteal_split.txt 2>&1
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal.txt 2>&1
timeout 900 python tools/ablation.py --next1 --scale 20 --workers 8 --out $O/abl_next1.json > $O/abl_next1.txt 2>&1
cat $O/abl_fsteal.txt $O/abl_fsteal_split.txt $O/abl_osteal.txt
echo done
