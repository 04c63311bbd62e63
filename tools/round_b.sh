mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -2 gpurun_out/pytest_gpu.log
for c in c2 c4 c3 c1; do
timeout 400 python bench.py --workload $c --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 1 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; echo bench $c rc=$?
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_pointwise" -c 6 -o gpurun_out/prof_c2b -f python tools/prof_run.py --workload c2 --schemes exact:0,center:2,row:2 --reps 2 > gpurun_out/ncu_c2b.log 2>&1; echo ncu rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_tiles" -c 2 -o gpurun_out/prof_c4b -f python tools/prof_run.py --workload c4 --schemes row:4,exact:0 --reps 1 > gpurun_out/ncu_c4b.log 2>&1; echo ncu rc=$?
du -sh gpurun_out
