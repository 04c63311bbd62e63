mkdir -p gpurun_out
for v in default runs occ3 runs_occ3; do
  if [ $v = default ]; then L=""; else L=$PWD/abtmp/lib_$v.so; fi
  PARAPROX_LIB=$L timeout 400 python tools/kbench.py --workloads c1,c2,c4,c3 --reps 10 > gpurun_out/kb_$v.jsonl 2>&1; echo kb $v rc=$?
done
PARAPROX_LIB=$PWD/abtmp/lib_runs.so timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_tiles" --csv --log-file gpurun_out/dram_runs.csv python tools/prof_run.py --workload c4 --schemes row:4,exact:0,row:1,col:4 --reps 1 > gpurun_out/ncu_runs.log 2>&1; echo ncu rc=$?
