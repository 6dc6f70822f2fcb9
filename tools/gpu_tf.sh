#!/bin/bash
# GPU-box helper: K3 tile-filter / chunk-key A/B (the experiment recorded in DESIGN.md §5; the code it
# drove was reverted, so at HEAD SKYCUBE_K3_TILEFILTER / SKYCUBE_K3_KEYSHIFT have no effect).  GPU tests first (TESTS=0 skips), then bench lines for
# CONFIGS under each (SKYCUBE_K3_TILEFILTER, SKYCUBE_K3_KEYSHIFT) pair in VARIANTS ("tf:shift ...").
mkdir -p gpurun_out
if [ "${TESTS:-1}" != 0 ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > gpurun_out/tf_tests.log
  cat gpurun_out/tf_tests.log
fi
for c in ${CONFIGS:-H}; do
  for v in ${VARIANTS:-0:0 1:0 1:8 1:10 1:12}; do
    tf=${v%%:*}; ks=${v##*:}
    SKYCUBE_K3_TILEFILTER=$tf SKYCUBE_K3_KEYSHIFT=$ks timeout 600 python bench.py --steps 3 --warmup 3 --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 > gpurun_out/tf_${c}_${tf}_${ks}.json
    python tools/bench_summary.py gpurun_out/tf_${c}_${tf}_${ks}.json "tf=$tf ks=$ks"
  done
done
