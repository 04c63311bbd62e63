python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -rf -p no:cacheprovider > gpurun_out/pytest_r02e.log 2>&1; echo pytest rc=$?; tail -4 gpurun_out/pytest_r02e.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_lattice|k_hotspot" -c 2 -o gpurun_out/prof_r02e -f python tools/prof_r02.py --only lattice,hotspot --reps 1 > gpurun_out/ncu_r02e.log 2>&1; echo ncu rc=$?
