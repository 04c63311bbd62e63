python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_lattice_gpu.py tests/test_hotspot_gpu.py tests/test_peer_gpu.py tests/test_parity_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -3
timeout 300 python tools/kbench.py --workloads c1,c2,c3,c4 > gpurun_out/kbench_r02d.jsonl 2>&1; echo kbench rc=$?
grep lattice gpurun_out/kbench_r02d.jsonl
timeout 300 python tools/hotspot.py --out gpurun_out/hotspot_r02d.json 2>&1 | grep 8192 | cut -c1-260
