#!/bin/bash
# Bench the step with several degridder variants: bash scripts/sweep_degridder2.sh NAME...
CFG=${CFG:-lofar}
TS=${TS:-0}
for V in "$@"; do
  echo "== $V"
  IDG_DEGRIDDER_VARIANT="$V" timeout 600 python bench.py --config $CFG --timesteps $TS --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --rho-iterations 2048 2>/dev/null \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print(f\"value {d['value']:.1f} grid {d['grid_mvis_s']:.1f} degrid {d['degrid_mvis_s']:.1f} MVis/s, gridder {k['gridder']['avg_ms']:.2f} ms ({k['gridder']['variant']}), degridder {k['degridder']['avg_ms']:.2f} ms ({k['degridder']['variant']}), clocks {d['clocks']['sm_mhz']}\")"
done
