// Block entry / exit instrumentation (K1) -- Paella Fig. 6 (PAPER.md P848-870, §4.1
// P872-899) re-designed for sm_100a:
//
//  * one elected thread per block does the counter atomic; the other warps never
//    wait on it at entry (they start computing immediately);
//  * per-launch counters {start, end} in device memory, slot = uid mod NCTR, never
//    reset -- the dispatcher passes the slot's running base (reading C2-Q1);
//  * the block whose count reaches a multiple of G or the grid total claims a ring
//    index with one atomicAdd on the tail (power-of-two ring + lap tag, C2-Q2/Q3) and
//    writes ONE 16-byte record {type, count, smid, uid | globaltimer, group} with a
//    single vector store straight into pinned, mapped host memory (P1104-1106);
//  * exit: __syncthreads (all outputs of the block written), a release fence
//    (an acq_rel end-counter atomic: gpu scope; system scope for a job's last kernel,
//    whose output lives in client host memory), so a successor kernel launched after
//    the dispatcher saw the final COMPLETION reads complete data (reading C2-Q19);
//  * %smid is re-read at exit (reading C2-Q4).
//
// Compiled out entirely in the uninstrumented twin (INSTR = false).
#pragma once
#include "common.h"

namespace paella {

__device__ __forceinline__ uint32_t smid_reg() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

__device__ __forceinline__ void put_record(const InstrArgs& ia, uint32_t type, uint32_t count_in_group,
                                           uint32_t group) {
  uint32_t idx = atomicAdd(ia.tail, 1u);
  uint32_t slot = idx & ia.mask;
  uint32_t lap = idx >> ia.log2cap;
  Rec r = rec_encode(type, count_in_group, smid_reg(), lap, ia.uid, globaltimer(), group);
  asm volatile("st.global.v2.u64 [%0], {%1, %2};" ::"l"(ia.ring + slot), "l"(r.w0), "l"(r.w1)
               : "memory");
}

// count = 1-based index of this block's arrival at the counter
__device__ __forceinline__ void maybe_record(const InstrArgs& ia, uint32_t type, uint32_t count,
                                             uint32_t total) {
  uint32_t G = ia.group;
  uint32_t r = count % G;
  if (r == 0 || count == total) {
    uint32_t n = (r == 0) ? G : r;
    put_record(ia, type, n, (count - 1) / G);
  }
}

// counter mode: this block's {start, end} counter pair (table blockid % NCTR_SUB)
__device__ __forceinline__ uint32_t* ctr_of_block(const InstrArgs& ia) {
  const uint32_t b = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  return ia.ctr + (b % NCTR_SUB) * ia.ctr_stride;
}

// T = the (1-D) thread that does the bookkeeping; kernels pick an otherwise idle
// thread so that compute never waits on the counter atomics
template <bool INSTR, uint32_t T = 0>
__device__ __forceinline__ void instr_enter(const InstrArgs& ia) {
  if constexpr (INSTR) {
    if (threadIdx.x == T && threadIdx.y == 0 && threadIdx.z == 0) {
      if (ia.flags & INSTR_CTR) {
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia)) : "memory");
      } else {
        uint32_t total = gridDim.x * gridDim.y * gridDim.z;
        uint32_t c = atomicAdd(&ia.ctr[0], 1u) + 1u - ia.base;
        maybe_record(ia, REC_PLACEMENT, c, total);
      }
    }
  }
}

// Programmatic dependent launch.  pdl_wait: block until the kernel this
// one was queued behind on its stream has completed and its memory is visible (a no-op
// for plain launches); every read of a predecessor's output and every output store
// comes after it.  pdl_trigger: this block no longer needs anything that a dependent's
// early start could disturb, so the dependent grid may be placed (its blocks run
// their independent prologue -- barrier init, TMEM allocation, weight prefetch -- and
// then pdl_wait).  Placement is still reported when blocks really start.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// SIMT kernels: bookkeeping, wait for the predecessor, then let the successor be
// placed right away (these kernels are short; the successor's prologue overlaps them)
template <bool INSTR>
__device__ __forceinline__ void kernel_begin(const InstrArgs& ia) {
  instr_enter<INSTR>(ia);
  pdl_wait();
  pdl_trigger();
}

// Counter mode, a job's LAST kernel (its output is the logits in client host memory):
// each block releases its outputs with a GPU-scope release reduction of the exit count.
// The host learns the count only through the mirror warp, which acquires it and issues a
// system-scope fence before publishing it (k_notify_mirror): that fence is cumulative
// over the logits the blocks released to it, so the host never sees the launch complete
// before every logit is visible -- one system-scope flush per batch of counter changes
// instead of one per block.  INSTR_SYSREL (experiment) restores the per-block
// system-scope release.
__device__ __forceinline__ void last_kernel_exit(const InstrArgs& ia) {
  if (ia.flags & INSTR_SYSREL)
    asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
  else
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
}

// exit count of a block whose every other thread is already past a CTA barrier (the
// caller is the block's last active thread): no second barrier
template <bool INSTR>
__device__ __forceinline__ void instr_exit_last_thread(const InstrArgs& ia) {
  if constexpr (INSTR) {
    if (ia.flags & INSTR_CTR) {
      if (ia.flags & INSTR_LAST)
        last_kernel_exit(ia);
      else if (ia.flags & INSTR_RELAXED)
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
      else
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
    } else {
      uint32_t old;
      if (ia.flags & INSTR_LAST)
        asm volatile("atom.acq_rel.sys.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&ia.ctr[1]) : "memory");
      else
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&ia.ctr[1]) : "memory");
      const uint32_t total = gridDim.x * gridDim.y * gridDim.z;
      maybe_record(ia, REC_COMPLETION, old + 1u - ia.base, total);
    }
  }
}

template <bool INSTR, uint32_t T = 0>
__device__ __forceinline__ void instr_exit(const InstrArgs& ia) {
  if constexpr (INSTR) {
    if ((ia.flags & (INSTR_CTR | INSTR_RELAXED)) == (INSTR_CTR | INSTR_RELAXED)) {
      // relaxed exit count (B200-Q4): it orders nothing (the job's data
      // dependencies ride on stream order), so no block barrier either -- the
      // bookkeeping thread counts the block when it gets here; the dispatcher may see
      // the block finished a few hundred ns before its last warp retires, which only
      // shifts the occupancy estimate
      if (threadIdx.x == T && threadIdx.y == 0 && threadIdx.z == 0)
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
      return;
    }
    __syncthreads();
    if (threadIdx.x == T && threadIdx.y == 0 && threadIdx.z == 0 && (ia.flags & INSTR_CTR)) {
      // counter mode: a release reduction (the block's outputs, ordered before it by the
      // barrier, are visible before the count is); nothing is waited for, the block
      // retires at once.  A job's last kernel: one system-scope flush per grid.
      if (ia.flags & INSTR_LAST)
        last_kernel_exit(ia);
      else if (ia.flags & INSTR_RELAXED)   // data dependencies ride on stream order
        asm volatile("red.relaxed.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
      else
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr_of_block(ia) + 1) : "memory");
    } else if (threadIdx.x == T && threadIdx.y == 0 && threadIdx.z == 0) {
      // acq_rel atomic: releases this block's outputs (ordered before by the barrier,
      // release is cumulative) and acquires the earlier blocks' before the record is
      // written; system scope for a job's last kernel, whose output is in host memory
      uint32_t old;
      if (ia.flags & INSTR_LAST)
        asm volatile("atom.acq_rel.sys.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&ia.ctr[1]) : "memory");
      else
        asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], 1;" : "=r"(old) : "l"(&ia.ctr[1]) : "memory");
      uint32_t total = gridDim.x * gridDim.y * gridDim.z;
      maybe_record(ia, REC_COMPLETION, old + 1u - ia.base, total);
    }
  }
}

}  // namespace paella
