#!/bin/bash
# GPU-box helper: bench lines for CONFIG under each environment assignment in VARIANTS (space-separated,
# "-" = none; e.g. VARIANTS="- SKYCUBE_K3_TPC=281"), then (TESTS=1) the GPU tests.
mkdir -p gpurun_out
if [ "${TESTS:-0}" != 0 ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
fi
for c in ${CONFIGS:-H}; do
  for v in ${VARIANTS:--}; do
    tag=$(echo "$v" | tr '=' '_')
    if [ "$v" = "-" ]; then envv=""; else envv="$v"; fi
    env $envv timeout 600 python bench.py --steps 5 --warmup 3 --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 > gpurun_out/eab_${c}_$tag.json
    python tools/bench_summary.py gpurun_out/eab_${c}_$tag.json "$v"
  done
done
