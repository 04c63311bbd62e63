mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$?
timeout 900 python -m pytest tests -m gpu -q --maxfail=30 > gpurun_out/pytest_gpu.log 2>&1; echo pytest rc=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 300 python bench.py > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err; echo bench rc=$?
timeout 400 python bench.py --workload c4 --steps 20 --warmup 3 --no-cpu-baseline --e2e-steps 2 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo bench c4 rc=$?
timeout 400 python tools/kbench.py > gpurun_out/kbench.jsonl 2>&1; echo kbench rc=$?
if [ -x abtmp/mapbench ]; then
  (./abtmp/mapbench 30 1 10; ./abtmp/mapbench 24 8 30) > gpurun_out/mapbench.jsonl 2>&1; echo mapbench rc=$?
fi
