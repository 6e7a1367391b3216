#!/bin/bash
# The paper's design space (Fig. 5 / Tables III-IV / V) on its own TMM (int32 4096^2, 32x32 thread-block
# regions, MOD+XOR), B200: store x lock x reduction.  -> gpurun_out/design_<workload>/*.json
# Usage: bash tools/design_space.sh [workload]   (default tmm4096_i32_paper; spmv4m = the paper's SPMV class)
WL=${1:-tmm4096_i32_paper}
D=gpurun_out/design_$WL
mkdir -p $D
for st in array quad_cas quad_lock cuckoo cuckoo_lock; do
  for sh in "" "--no-shuffle"; do
    tag=${st}${sh:+_noshfl}
    timeout 900 python bench.py --workload $WL --store $st $sh --steps 3 --warmup 3 --overhead-reps 10 \
      --no-cpu-baseline > $D/$tag.json 2> $D/$tag.err || tail -2 $D/$tag.err
  done
done
D=$D python - <<'PY'
import glob, json, os
print("| store | reduction | t_prot ms | t_unprot ms | LP overhead (median of pairs) | pair IQR | slowdown (x) | "
      "hash collisions (quad: extra probes; cuckoo: evictions) |")
print("|---|---|---|---|---|---|---|---|")
for f in sorted(glob.glob(os.environ["D"] + "/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    c = d["config"]
    iqr = d.get("lp_overhead_detail", {}).get("iqr_pct", [None, None])
    print(f"| {c['store']} | {c['reduction']} | {d['t_protected_ms']:.3f} | {d['t_unprotected_ms']:.3f} | "
          f"{d['lp_overhead_pct']:+.2f}% | [{iqr[0]:+.2f}, {iqr[1]:+.2f}]% | "
          f"{d['t_protected_ms'] / d['t_unprotected_ms']:.2f} | {d.get('hash_collisions')} |")
PY
