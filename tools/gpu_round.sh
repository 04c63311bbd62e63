#!/bin/bash
# One GPU round: smoke, GPU tests, bench lines for every workload, ncu launch
# list of the default bench command and a full capture of the top kernels.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 900 python -m pytest tests -m gpu -q --maxfail=30 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo bench rc=$?
for c in c1 c3 c4; do
  timeout 400 python bench.py --workload $c --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo bench $c rc=$?
done
if [ -z "$NO_NCU" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/ncu_launches.log 2>&1; echo ncu-launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_pointwise|k_lattice|k_quality_flat" -c 12 -o gpurun_out/prof_c2 -f python tools/prof_run.py --workload c2 --schemes exact:0,center:2,row:1 --lattice row:1,row:4 --quality --reps 2 > gpurun_out/ncu_c2.log 2>&1; echo ncu rc=$?
fi
cat gpurun_out/bench_c2.json
timeout 900 python tools/toq_sweep.py > gpurun_out/toq_sweep.log 2>&1; echo sweep rc=$?
timeout 400 python tools/kbench.py > gpurun_out/kbench.jsonl 2>&1; echo kbench rc=$?
timeout 600 python tools/convsep.py > gpurun_out/convsep.log 2>&1; echo convsep rc=$?
timeout 600 python tools/hotspot.py > gpurun_out/hotspot.log 2>&1; echo hotspot rc=$?
if [ -z "$NO_NCU" ]; then
for c in c1 c3 c4; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_pointwise|k_lattice" -c 4 -o gpurun_out/prof_$c -f python tools/prof_run.py --workload $c --schemes exact:0,center:9 --reps 1 > gpurun_out/ncu_$c.log 2>&1; echo ncu $c rc=$?
done
fi
[ -z "$NO_NCU" ] && bash tools/ncu_bytes.sh
bash tools/sanitize.sh
# summarise the ncu captures here on the box (gpurun_out/ must stay < 64 MiB)
for c in c1 c2 c3 c4; do
  if [ -f gpurun_out/prof_$c.ncu-rep ]; then
    python tools/ncu_summary.py full gpurun_out/prof_$c.ncu-rep --workload $c --traffic gpurun_out/traffic_box.json > gpurun_out/ncu_full_$c.md 2>/dev/null
    rm -f gpurun_out/prof_$c.ncu-rep
  fi
done
python tools/ncu_summary.py launches gpurun_out/launches_c2.csv > gpurun_out/launches_c2.md 2>/dev/null
python tools/ncu_summary.py bytes gpurun_out/ncu_bytes_c2.csv gpurun_out/ncu_bytes_c4.csv > gpurun_out/ncu_bytes.md 2>/dev/null
du -sh gpurun_out

