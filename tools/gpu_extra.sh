#!/bin/bash
# A/B of tile-kernel occupancy, sanitizers, per-workload ncu captures.
mkdir -p gpurun_out
timeout 400 python tools/kbench.py > gpurun_out/kb_cur.jsonl 2>&1; echo kb cur rc=$?
PARAPROX_LIB=$PWD/build/ab/libparaprox_occ3.so timeout 400 python tools/kbench.py > gpurun_out/kb_occ3.jsonl 2>&1; echo kb occ3 rc=$?
bash tools/sanitize.sh
for c in c1 c3 c4; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_pointwise|k_lattice" -c 4 -o gpurun_out/prof_$c -f python tools/prof_run.py --workload $c --schemes exact:0,center:9 --reps 1 > gpurun_out/ncu_$c.log 2>&1; echo ncu $c rc=$?
done
timeout 300 python bench.py --steps 50 --warmup 5 --no-cpu-baseline > gpurun_out/bench_c2_e2e.json 2>&1; echo bench rc=$?
