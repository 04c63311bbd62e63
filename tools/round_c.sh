mkdir -p gpurun_out
for pr in 0 128 256; do
  PARAPROX_TMA_L2PROMO=$pr timeout 400 python tools/kbench.py --workloads c2,c4,c3 --reps 10 > gpurun_out/kb_promo$pr.jsonl 2>&1; echo kb $pr rc=$?
done
for pr in 0 256; do
PARAPROX_TMA_L2PROMO=$pr timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:"k_tiles" --csv --log-file gpurun_out/dram_promo$pr.csv python tools/prof_run.py --workload c4 --schemes row:4,exact:0,row:1,col:4 --reps 1 > /dev/null 2>&1; echo ncu $pr rc=$?
done
