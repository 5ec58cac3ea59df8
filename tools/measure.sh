#!/bin/bash
# Round measurement script (one parameterised replacement for the per-session scripts of round 1): bench lines
# of the configs given in CONFIGS (default C1..C5 + delta-PR), each copied to $O/bench_<C>[_<alg>].json with a
# one-line summary. Run under gpurun; O defaults to gpurun_out/measure.
#   CONFIGS="C2 C5" O=gpurun_out/m bash tools/measure.sh
O=${O:-gpurun_out/measure}; mkdir -p $O
CONFIGS=${CONFIGS:-"C2 C1 C3 C4 C5 C5:dpr"}
for spec in $CONFIGS; do
  cfg=${spec%%:*}; alg=""; [ "$spec" != "$cfg" ] && alg=${spec#*:}
  name=$cfg${alg:+_$alg}
  args="--config $cfg ${alg:+--alg $alg}"
  case $cfg in
    C1) args="$args --steps 50" ;;
    C3) args="$args --steps 3 --warmup 3 --no-e2e" ;;
    C4) args="$args --steps 5 --warmup 3 --no-e2e" ;;
    C5) args="$args --steps 3 --warmup 3 --no-e2e" ;;
  esac
  timeout 1500 python bench.py $args > $O/bench_$name.json 2> $O/bench_$name.err; echo "$name rc=$?"
  python - "$O/bench_$name.json" "$name" <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
    r = d.get("roofline") or {}
    p = (d.get("detail") or {}).get("parity_full_size") or {}
    print(sys.argv[2], d["value"], d["unit"], d["ms_per_step"], "ms;", r.get("kernel"), r.get("achieved"), "GB/s frac", r.get("frac"),
          "; parity", p.get("exact"), p.get("rule"), "; e2e", (d.get("e2e") or {}).get("value"), "; cpu", (d.get("cpu_baseline") or {}).get("value"),
          "; clocks", d.get("clocks"))
except Exception as e:
    print(sys.argv[2], "no line:", e)
PY
done
