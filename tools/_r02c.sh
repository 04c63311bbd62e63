python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_fullsize_tuner_gpu.py -q -rf -p no:cacheprovider 2>&1 | tail -3
s=$(date +%s.%N); python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench_r02_default.json 2> gpurun_out/bench_r02_default.err; echo bench rc=$? wall=$(echo "$(date +%s.%N) - $s" | bc)
s=$(date +%s.%N); python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_r02_ref.json 2> gpurun_out/bench_r02_ref.err; echo ref rc=$? wall=$(echo "$(date +%s.%N) - $s" | bc)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tiles|k_lattice|k_hotspot" -c 6 -o gpurun_out/prof_r02a -f python tools/prof_r02.py --reps 1 > gpurun_out/ncu_r02a.log 2>&1; echo ncu rc=$?
ls -la gpurun_out/prof_r02a.ncu-rep
