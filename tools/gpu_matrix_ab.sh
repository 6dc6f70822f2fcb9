#!/bin/bash
# GPU-box helper: bench lines for every (library, environment) pair: LIBS x VARIANTS x CONFIGS.
mkdir -p gpurun_out
P=paper_conf_sigmod_boghcsa17_b200
for c in ${CONFIGS:-H}; do
  for l in ${LIBS:-libskycube.so}; do
    for v in ${VARIANTS:--}; do
      if [ "$v" = "-" ]; then envv=""; else envv="$v"; fi
      env $envv SKYCUBE_LIB=$PWD/$P/$l timeout 600 python bench.py --steps ${STEPS:-5} --warmup 3 --config $c --no-e2e --no-cpu 2>/dev/null | tail -1 > gpurun_out/mab.json
      python tools/bench_summary.py gpurun_out/mab.json "$l $v" | cut -c1-170
    done
  done
done
