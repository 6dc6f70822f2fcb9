#!/bin/bash
# GPU-box helper: the round's evidence in one call -- GPU tests, smoke, bench lines for every BASELINE
# config (+ HashCube output, SDSC comparator, reference arm sample), the ncu launch list of the default
# bench, and --set full captures of the top kernels.  Everything lands in gpurun_out/ev_*.
mkdir -p gpurun_out
python -c "from paper_conf_sigmod_boghcsa17_b200 import build; build.build()"
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/ev_gpu.txt
timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -4 > gpurun_out/ev_tests.log
python __graft_entry__.py smoke > gpurun_out/ev_smoke.log 2>&1
for c in H C3A C3I C3C C2 C5 C4; do
  timeout 900 python bench.py --config $c --cpu-seconds ${CPU_S:-12} 2>/dev/null | tail -1 > gpurun_out/ev_bench_$c.json
done
timeout 600 python bench.py --output hashcube --cpu-seconds 2 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_hashcube.json
timeout 600 python bench.py --config C2 --algo sdsc --steps 3 2>/dev/null | tail -1 > gpurun_out/ev_bench_C2_sdsc.json
timeout 600 python bench.py --config C3I --algo sdsc --steps 1 2>/dev/null | tail -1 > gpurun_out/ev_bench_C3I_sdsc.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_reference.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_H.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ev_ncu_launch.log 2>&1
for spec in "H:k3_mdmc" "H:k1_prefilter" "C5:k3_owner" "C4:k3_mdmc"; do
  cfg=${spec%%:*}; k=${spec##*:}
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -c 1 -f -o gpurun_out/ev_prof_${k}_$cfg \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config $cfg > gpurun_out/ev_ncu_${k}_$cfg.log 2>&1
done
# summaries on the box (gpurun_out/ comes back only if it stays under 64 MiB): keep one full report
python tools/evidence_summary.py ${TAG:-r01} gpurun_out/ev_out
cp gpurun_out/ev_prof_k3_mdmc_H.ncu-rep gpurun_out/ev_out/ 2>/dev/null
rm -f gpurun_out/ev_prof_*.ncu-rep
du -sh gpurun_out
cat gpurun_out/ev_tests.log gpurun_out/ev_smoke.log
for f in gpurun_out/ev_bench_*.json; do echo "$f: $(head -c 300 $f)"; done
