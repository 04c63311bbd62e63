python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_r02b.log 2>&1; echo pytest rc=$?; tail -8 gpurun_out/pytest_r02b.log
/usr/bin/time -v python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_r02_default.json 2> gpurun_out/bench_r02_default.err; echo bench rc=$?
grep -E "Elapsed|Maximum resident" gpurun_out/bench_r02_default.err
timeout 400 python bench.py --workload c2 --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench_r02_c2.json 2> gpurun_out/bench_r02_c2.err; echo bench c2 rc=$?
/usr/bin/time -v python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_r02_ref.json 2> gpurun_out/bench_r02_ref.err; echo ref rc=$?
grep -E "Elapsed" gpurun_out/bench_r02_ref.err
