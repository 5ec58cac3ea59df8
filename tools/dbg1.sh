O=gpurun_out/dbg1; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_units.py -q -k online_p > $O/p.log 2>&1; echo "p rc=$?"; tail -3 $O/p.log; grep -E "^E  " $O/p.log | head -10
python - <<'PY'
import sys; sys.path.insert(0, '.')
import inputs
from tests.gpu_helpers import gpu_run
g = inputs.grid(256, seed=9)
for kw in (dict(num_gpus=4, split_units=True), dict(num_gpus=8, split_units=True), dict(num_gpus=4)):
    out, st, _ = gpu_run(g, "sssp", 0, osteal="cost", osteal_sync_edges=0.0, tail_vertices=0, **kw)
    print(kw, "p", st.osteal_p, "samples", st.osteal_p_samples, "owners", st.final_owners, "ms", st.ms, "iters", st.iterations, "bar", st.unit_barriers)
    out, st, _ = gpu_run(g, "sssp", 0, osteal=False, tail_vertices=0, **kw)
    print("   no osteal ms", st.ms)
PY
