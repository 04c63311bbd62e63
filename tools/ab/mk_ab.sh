# A/B builds: copy csrc, apply patch scripts (e.g. tools/ab/trace_patch.py), build abship/lib_<name>.so;
# on the GPU box load it with PARAPROX_LIB=$PWD/abship/lib_<name>.so (abship/ is git-ignored, not gpurun-ignored)
# tools/ab/mk_ab.sh <name> [patch.py ...]: copy csrc, apply patches, build abship/lib_<name>.so
set -e
n=$1; shift
R=/root/repo
rm -rf $R/build/ab_$n && mkdir -p $R/build/ab_$n/pkg $R/build/ab_$n/include
cp -r $R/paper_conf_asplos_samadijlm14_b200/csrc $R/build/ab_$n/pkg/csrc && cp $R/include/paraprox.h $R/build/ab_$n/include/
for p in "$@"; do python $p $R/build/ab_$n/pkg/csrc; done
cd $R/build/ab_$n/pkg/csrc && make -j8 OUT=$R/abship/lib_$n.so OBJDIR=$R/build/ab_$n/obj 2>&1 | grep -E "error" || true
ls -la $R/abship/lib_$n.so
