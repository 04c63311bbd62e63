#!/bin/bash
# A/B of library builds on the GPU box: kbench for the in-tree library and for
# every abtmp/lib_<name>.so given, into gpurun_out/kb_<tag>_<name>.jsonl.
#   (here)  make -C paper_conf_asplos_samadijlm14_b200/csrc OUT=$PWD/abtmp/lib_x.so OBJDIR=$PWD/build/ab_x EXTRA="-D..."
#   (box)   bash tools/ab_kbench.sh <tag> x [y ...]   -> python tools/abcmp.py gpurun_out/kb_<tag>_default.jsonl ...
mkdir -p gpurun_out
tag=$1; shift
for v in default "$@"; do
  if [ $v = default ]; then L=""; else L=$PWD/abtmp/lib_$v.so; fi
  PARAPROX_LIB=$L timeout 400 python tools/kbench.py --workloads ${WORKLOADS:-c1,c2,c4,c3} --reps 10 > gpurun_out/kb_${tag}_$v.jsonl 2>&1
  echo "kb $v rc=$?"
done
