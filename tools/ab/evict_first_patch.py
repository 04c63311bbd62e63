"""A/B patch: TMA output stores with an L2 evict_first cache policy (the
output of a launch does not linger dirty in L2 for the next launch to evict)."""
import sys
d = sys.argv[1]
p = d + "/tma.cuh"
s = open(p).read()
old = '''    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                     reinterpret_cast<uint64_t>(map)),
                 "r"(smem_u32(smem)), "r"(x), "r"(y), "r"(z)
                 : "memory");'''
new = '''    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3, %4}], [%1], %5;" ::"l"(
                     reinterpret_cast<uint64_t>(map)),
                 "r"(smem_u32(smem)), "r"(x), "r"(y), "r"(z), "l"(pol)
                 : "memory");'''
assert old in s
open(p, "w").write(s.replace(old, new))
