for v in default ef; do
  if [ $v = default ]; then L=""; else L=$PWD/abship/lib_$v.so; fi
  PARAPROX_LIB=$L timeout 300 python tools/launch_overhead.py --out gpurun_out/lo_n_$v.json > gpurun_out/lo_n_$v.log 2>&1; grep fixed gpurun_out/lo_n_$v.log
  PARAPROX_LIB=$L timeout 300 python tools/kbench.py --workloads c1,c2,c4,c3 --reps 20 > gpurun_out/kb_n_$v.jsonl 2>&1
done
