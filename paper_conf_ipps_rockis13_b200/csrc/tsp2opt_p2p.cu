// tsp2opt_p2p.cu -- the per-sweep allreduce-min of the packed best-move key
// over PEER MEMORY instead of NCCL.
//
// PAPER.md L18 §VI: "dividing the 2-opt task between multiple devices".  Each
// rank owns a mailbox in its own HBM, exported with cudaIpcGetMemHandle and
// mapped by every other rank (cudaIpcOpenMemHandle: NVLink / NVSwitch peer
// memory across GPUs, or the same HBM for ranks sharing one GPU).  After its
// shard's sweep a rank STORES its key into every peer's mailbox (one 8-byte
// store per peer, then a system-scope fence and the sequence number), spins on
// its own mailbox until every rank's key of this sweep has arrived, and writes
// the minimum into its slot -- the same value on every rank, so every rank
// applies the same reversal and the replicated state stays bit-identical.
// Mailboxes are double-buffered by sequence parity: a peer can run at most one
// exchange ahead (it needs this rank's next key to go further), so it never
// overwrites a key this rank has not read yet.  One 32-thread block; no NCCL
// launch latency, one store per peer and one poll per rank.
#include "tsp2opt_device.cuh"
#include "tsp2opt_internal.h"

namespace tsp2opt {

__global__ void p2p_min_kernel(Slot* __restrict__ slot, Mailbox* const* __restrict__ peers, int rank, int world,
                               int respect_done, long long timeout_cycles)
{
    pdl_trigger();
    pdl_wait();
    __shared__ unsigned long long s_key[kP2PMaxWorld];
    __shared__ int s_state;  // 0 run, 1 skip (converged), 2 timeout
    __shared__ unsigned long long s_seq;
    Mailbox* me = peers[rank];
    const int t = threadIdx.x;
    if (t == 0) {
        s_state = (respect_done && *(volatile int*)&slot->done) ? 1 : 0;  // identical on every rank
        s_seq = *(volatile unsigned long long*)&me->counter + 1;
    }
    __syncthreads();
    if (s_state) return;
    const unsigned long long s = s_seq;
    const int par = (int)(s & 1);
    const unsigned long long key = *(volatile unsigned long long*)&slot->key;
    if (t < world) {  // publish: key, then (after a system-scope fence) the sequence number
        Mailbox* p = peers[t];
        *(volatile unsigned long long*)&p->key[par][rank] = key;
        __threadfence_system();
        *(volatile unsigned long long*)&p->seq[par][rank] = s;
    }
    if (t < world) {  // collect rank t's key of this exchange from the own mailbox
        const long long t0 = clock64();
        while (*(volatile unsigned long long*)&me->seq[par][t] != s) {
            if (clock64() - t0 > timeout_cycles) {
                s_state = 2;
                break;
            }
            __nanosleep(64);
        }
        __threadfence();
        s_key[t] = *(volatile unsigned long long*)&me->key[par][t];
    }
    __syncthreads();
    if (t == 0) {
        if (s_state == 2) {
            atomicOr(&slot->done, kDoneExchangeTimeout);
            return;
        }
        unsigned long long m = s_key[0];
        for (int r = 1; r < world; r++) m = s_key[r] < m ? s_key[r] : m;
        slot->key = m;
        me->counter = s;
    }
}

cudaError_t launch_p2p_min(Slot* slot, Mailbox* const* peers, int rank, int world, int respect_done,
                           cudaStream_t st)
{
    const long long timeout = 30LL * 2000000000LL;  // ~30 s at 2 GHz: a peer that never arrives
    cudaError_t e = launch_kernel_pdl(p2p_min_kernel, dim3(1), dim3(32), 0, st, slot, peers, rank, world,
                                      respect_done, timeout);
    count_launch(1);
    return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace tsp2opt
