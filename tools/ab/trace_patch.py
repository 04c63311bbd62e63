import sys
d = sys.argv[1]
def sub(p, old, new):
    p = d + '/' + p
    s=open(p).read(); assert old in s, (p, old[:60]); s=s.replace(old,new,1); open(p,'w').write(s)
p='k_tiles.cuh'
sub(p,'''namespace ppx {

constexpr int kTW = 128;''','''namespace ppx {
__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
__device__ __forceinline__ unsigned smid_() {
    unsigned r;
    asm volatile("mov.u32 %0, %smid;" : "=r"(r));
    return r;
}

constexpr int kTW = 128;''')
sub(p,'''    const int tid = threadIdx.x, lane = tid & 31, wi = tid >> 5;
    const int tiles_per_frame = A.tiles_x * A.tiles_y;

    auto coords''','''    const int tid = threadIdx.x, lane = tid & 31, wi = tid >> 5;
    const int tiles_per_frame = A.tiles_x * A.tiles_y;
    unsigned long long* TR = (!Q && A.part && blockIdx.x < 65536) ? reinterpret_cast<unsigned long long*>(A.part) + 8ull * blockIdx.x : nullptr;
    if (tid == 0 && TR) TR[0] = gtime();

    auto coords''')
sub(p,'''    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    // the CTA's k-th tile''','''    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    if (tid == 0 && TR) TR[1] = gtime();
    // the CTA's k-th tile''')
sub(p,'''        mbar_wait(&bars[s], (it / G::STAGES) & 1);
''','''        mbar_wait(&bars[s], (it / G::STAGES) & 1);
        if (it == 0 && tid == 0 && TR) TR[2] = gtime();
''')
sub(p,'''        __syncthreads();  // stage s fully consumed before it is refilled
    }''','''        __syncthreads();  // stage s fully consumed before it is refilled
        if (it == 0 && tid == 0 && TR) TR[3] = gtime();
    }''')
sub(p,'''    if (A.tma_store && tid == 0) bulk_wait_all();''','''    if (A.tma_store && tid == 0) bulk_wait_all();
    if (tid == 0 && TR) {
        TR[4] = gtime();
        TR[5] = smid_();
        TR[6] = it;
    }''')
p='dispatch.cu'
sub(p,'''    A.part = qo ? qo->part : nullptr;''','''    static void* trace_buf = nullptr;
    if (!trace_buf) cudaMalloc(&trace_buf, 65536 * 8 * 8);
    A.part = qo ? qo->part : (double*)trace_buf;
    g_trace_ptr = trace_buf;''')
sub(p,'''namespace ppx {

cudaError_t launch_generic(''','''namespace ppx {
void* g_trace_ptr = nullptr;

cudaError_t launch_generic(''')
sub(p,'''}  // namespace ppx
''','''}  // namespace ppx

extern "C" __attribute__((visibility("default"))) int paraprox_debug_trace(unsigned long long* h, int n) {
    if (!ppx::g_trace_ptr) return -1;
    return (int)cudaMemcpy(h, ppx::g_trace_ptr, 8ull * 8 * n, cudaMemcpyDeviceToHost);
}
''')
