#!/bin/bash
# GPU-box helper: GPU tests, then bench lines for CONFIGS under each K3 design (A, O), then (NCU=1) an ncu
# capture of K3 at H with the default design.
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()"
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > gpurun_out/ab_tests.log
cat gpurun_out/ab_tests.log
for c in ${CONFIGS:-H}; do
  for des in ${DESIGNS:-A O}; do
    SKYCUBE_K3_DESIGN=$des timeout 600 python bench.py --steps 3 --warmup 3 --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 > gpurun_out/ab_${c}_$des.json
    python tools/bench_summary.py gpurun_out/ab_${c}_$des.json $des
  done
done
if [ -n "$NCU" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KERNEL:-k3_} -c 1 -f -o gpurun_out/ab_prof \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config ${NCU_CFG:-H} > gpurun_out/ab_ncu.log 2>&1
  tail -2 gpurun_out/ab_ncu.log
fi
