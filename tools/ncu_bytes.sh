#!/bin/bash
# DRAM bytes per launch of the exact stencil, the tuned per-window
# approximation and the row lattice (NEXT-1) at c2 and c4 (ncu, cold L2 per
# kernel): the lattice is the variant that removes DRAM bytes.  Output:
# gpurun_out/ncu_bytes_<wl>.csv, summarised by tools/ncu_summary.py bytes.
mkdir -p gpurun_out
for wl in c2 c4; do
  sc="exact:0,center:2"; [ $wl = c4 ] && sc="exact:0,center:4"
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:"k_tiles|k_pointwise|k_lattice" --csv python tools/prof_run.py --workload $wl --schemes $sc \
    --lattice row:1,row:2,row:4 --reps 1 > gpurun_out/ncu_bytes_$wl.csv 2> gpurun_out/ncu_bytes_$wl.err
  echo "ncu bytes $wl rc=$?"
done
