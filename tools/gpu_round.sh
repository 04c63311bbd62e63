#!/bin/bash
# One GPU round (r02): smoke, GPU tests, the default bench line (c3, the
# driver's command) and the other workloads, the ncu launch list of the
# default bench command, ncu --set full of the c3 kernels (steady-state DRAM
# traffic: c3's 8.5 GB input is 67x L2), DRAM bytes exact / approximation /
# lattice, the c5 TOQ sweep, ConvSep, HotSpot, kbench, sanitizers.
# Everything lands in gpurun_out/ (< 64 MiB: ncu reports are summarised here).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 1200 python -m pytest tests -m gpu -q --maxfail=30 -p no:cacheprovider ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo bench rc=$?
timeout 600 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; echo ref rc=$?
for c in c1 c2 c4; do
  timeout 600 python bench.py --workload $c --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 5 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo bench $c rc=$?
done
if [ -z "$NO_NCU" ]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches_c3.csv \
    python bench.py --steps 20 --warmup 5 --no-cpu-baseline --e2e-steps 1 --reps 1 > gpurun_out/ncu_launches.log 2>&1; echo ncu-launches rc=$?
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_pointwise" -c 3 -o gpurun_out/prof_c3 -f \
    python tools/prof_run.py --workload c3 --schemes center:3,center:1 --reps 1 > gpurun_out/ncu_c3.log 2>&1; echo ncu c3 rc=$?
  bash tools/ncu_bytes.sh
fi
timeout 1200 python tools/toq_sweep.py > gpurun_out/toq_sweep.log 2>&1; echo sweep rc=$?
timeout 600 python tools/kbench.py --workloads c1,c2,c3,c4 --reps 20 > gpurun_out/kbench.jsonl 2>&1; echo kbench rc=$?
timeout 600 python tools/convsep.py > gpurun_out/convsep.log 2>&1; echo convsep rc=$?
timeout 600 python tools/hotspot.py > gpurun_out/hotspot.log 2>&1; echo hotspot rc=$?
timeout 600 python tools/launch_overhead.py > gpurun_out/launch_overhead.log 2>&1; echo launch-overhead rc=$?
# compute-sanitizer: closed on the GPU pool since the r02 final round (tools/sanitize.sh; r02_sanitizers.md
# is the last run, all four tools clean)
# summarise the ncu captures here on the box (gpurun_out/ must stay < 64 MiB)
if [ -f gpurun_out/prof_c3.ncu-rep ]; then
  python tools/ncu_summary.py full gpurun_out/prof_c3.ncu-rep --workload c3 --traffic gpurun_out/traffic_box.json > gpurun_out/ncu_full_c3.md 2>/dev/null
  (cd tools && python ncu_kernels.py ../gpurun_out/prof_c3.ncu-rep > ../gpurun_out/ncu_kernels_c3.md 2>/dev/null)
  rm -f gpurun_out/prof_c3.ncu-rep
fi
python tools/ncu_summary.py launches gpurun_out/launches_c3.csv > gpurun_out/launches_c3.md 2>/dev/null
python tools/ncu_summary.py bytes gpurun_out/ncu_bytes_c2.csv gpurun_out/ncu_bytes_c4.csv > gpurun_out/ncu_bytes.md 2>/dev/null
du -sh gpurun_out
