#!/bin/bash
# GPU-box helper: a lighter tools/gpu_evidence.sh (no SDSC lines, one --set full capture: K3 at H), for a
# refresh of the round's evidence at HEAD.  Summaries land in gpurun_out/ev_out (TAG prefix).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/ev_gpu.txt
timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -4 > gpurun_out/ev_tests.log
python __graft_entry__.py smoke > gpurun_out/ev_smoke.log 2>&1
for c in H C3A C3I C3C C2 C5 C4; do
  timeout 600 python bench.py --config $c --cpu-seconds ${CPU_S:-8} 2>/dev/null | tail -1 > gpurun_out/ev_bench_$c.json
done
timeout 600 python bench.py --output hashcube --cpu-seconds 2 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_hashcube.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 2>/dev/null | tail -1 > gpurun_out/ev_bench_H_reference.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev_launches_H.csv \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > gpurun_out/ev_ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k3_mdmc -c 1 -f -o gpurun_out/ev_prof_k3_mdmc_H \
  python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --config H > gpurun_out/ev_ncu_k3_mdmc_H.log 2>&1
python tools/evidence_summary.py ${TAG:-r01_final} gpurun_out/ev_out
rm -f gpurun_out/ev_prof_*.ncu-rep
cat gpurun_out/ev_tests.log gpurun_out/ev_smoke.log
for f in gpurun_out/ev_bench_*.json; do echo "$f: $(head -c 200 $f)"; done
