// Internal definitions shared by the host runtime and the device kernels of the
// CUDA path (never by the oracle).
//
// Notification record (readings C2-Q3/Q4/Q5 in DESIGN.md).
// The paper's entry is one 64-bit word {type:8, smId:8, kernId:32} (P1126-1133);
// we keep those fields and use a 16-byte record written with ONE vector store so
// it carries the block count, the group index, %globaltimer and a lap tag that
// detects torn / stale reads without an INVALID reset race:
//   w0 = type:8 | count:8 | smid:8 | tag:8 | uid:32
//   w1 = gtimer_ns:40 | group:16 | tag:8          tag = 0x80 | (lap & 0x7f)
// where lap = ring index >> log2(capacity).  type 0 = INVALID (P1110-1113).
#pragma once
#include <stdint.h>
#include <stddef.h>

#ifndef __CUDACC__
#define PAELLA_HD
#else
#define PAELLA_HD __host__ __device__
#endif

namespace paella {

enum : uint32_t { REC_INVALID = 0, REC_PLACEMENT = 1, REC_COMPLETION = 2 };

struct alignas(16) Rec {
  uint64_t w0, w1;
};

PAELLA_HD inline uint32_t rec_tag(uint32_t lap) { return 0x80u | (lap & 0x7fu); }

PAELLA_HD inline Rec rec_encode(uint32_t type, uint32_t count, uint32_t smid, uint32_t lap,
                                uint32_t uid, uint64_t gtimer, uint32_t group) {
  uint64_t tag = rec_tag(lap);
  Rec r;
  r.w0 = (uint64_t)(type & 0xff) | ((uint64_t)(count & 0xff) << 8) | ((uint64_t)(smid & 0xff) << 16) |
         (tag << 24) | ((uint64_t)uid << 32);
  r.w1 = (gtimer & ((1ull << 40) - 1)) | ((uint64_t)(group & 0xffff) << 40) | (tag << 56);
  return r;
}

struct RecFields {
  uint32_t type, count, smid, tag0, uid, group, tag1;
  uint64_t gtimer;
};

PAELLA_HD inline RecFields rec_decode(uint64_t w0, uint64_t w1) {
  RecFields f;
  f.type = (uint32_t)(w0 & 0xff);
  f.count = (uint32_t)((w0 >> 8) & 0xff);
  f.smid = (uint32_t)((w0 >> 16) & 0xff);
  f.tag0 = (uint32_t)((w0 >> 24) & 0xff);
  f.uid = (uint32_t)(w0 >> 32);
  f.gtimer = w1 & ((1ull << 40) - 1);
  f.group = (uint32_t)((w1 >> 40) & 0xffff);
  f.tag1 = (uint32_t)(w1 >> 56);
  return f;
}

// Per-launch instrumentation arguments (Fig. 6's extra parameters notifQ, kernId,
// P887-895, plus the per-launch counter slot -- reading C2-Q1).
// INSTR_CTR (counter mode): the block only bumps its launch's {start,
// end} counters with fire-and-forget reductions and writes no record; the mirror warp
// (k_notify_mirror) copies the counters to pinned host memory and the dispatcher turns
// counter progress into the same group-of-G records (engine.cpp::drain_counters)
enum : uint32_t { INSTR_ON = 1u, INSTR_LAST = 2u, INSTR_CTR = 4u, INSTR_RELAXED = 8u, INSTR_SYSREL = 16u };

struct InstrArgs {
  Rec* ring;          // device-visible pointer to the pinned, mapped ring
  uint32_t* tail;     // device counter: next ring index
  uint32_t* ctr;      // {start, end} block counters of this launch's slot (uid mod NCTR)
  uint32_t mask;      // capacity - 1
  uint32_t log2cap;
  uint32_t base;      // counter value of the slot before this launch (never reset)
  uint32_t uid;       // unique launch id (kernel id of the paper)
  uint32_t group;     // G
  uint32_t flags;     // INSTR_*
  uint32_t ctr_stride;   // counter mode: words between the NCTR_SUB counter tables
};

constexpr uint32_t NCTR = 4096;   // counter slots; > max in-flight launches (<= P)
constexpr uint32_t NCTR_M = 256;  // counter-mode slots (free list; > P x (lookahead + 1))
// counter mode: each launch's {start, end} counts are split over NCTR_SUB tables (block b
// counts in table b % NCTR_SUB, ctr_stride words apart) so the blocks of one launch do not
// all reduce into one L2 address; the host sums the tables
constexpr uint32_t NCTR_SUB = 4;

// Kernel-side arguments of one layer.  Activations are NHWC with an explicit
// channel stride/offset so that a concat is just producers writing into disjoint
// channel ranges of one buffer (zero-copy concat).
enum : uint32_t {
  LF_PROLOGUE = 1u,   // relu(scale*x + shift) on the input (DenseNet pre-activation)
  LF_CEIL = 2u,       // maxpool ceil mode
  LF_FINAL = 4u,      // output is the fp32 logits in client memory
  LF_RESIDUAL = 8u,
  LF_TRACE = 16u,     // debug: per-CTA phase timestamps (globaltimer) into trace
  LF_SPLIT_DSMEM = 32u,   // split-K reduced over DSMEM (round-2 design, A/B) instead of in L2
  LF_SPLIT_NOROT = 64u,   // (A/B) L2 split-K: every CTA reduces its rows in tile order
  LF_SPLIT_RELBAR = 128u, // (A/B) L2 split-K: release/acquire cluster barrier instead of a
                          // relaxed one after the reducing thread's own fence
  LF_MBAR_SPIN = 256u,    // (A/B) conv k-block loop: mbarrier.test_wait spin instead of try_wait
  LF_TMA_B = 512u,        // tcgen05 conv: B (activations) by TMA im2col (bmap) instead of the
                          // LDGSTS gather (cin % 64 == 0, no prologue)
};

struct LayerArgs {
  const void* in;       // NHWC, element type of the model (ingest: fp32 NCHW client memory)
  void* out;
  const void* res;      // residual (same layout as out)
  const void* w;        // packed weights (layout depends on the kernel)
  const float* bias;    // [cout] fp32
  const float* pro_scale;
  const float* pro_shift;
  uint32_t in_cs, in_co;    // channel stride / offset of the input buffer
  uint32_t out_cs, out_co;
  uint32_t res_cs, res_co;
  uint32_t cin, h, w_;      // input (channels used, H, W)
  uint32_t cout, oh, ow;
  uint32_t kh, kw, sh, sw, ph, pw, groups;
  uint32_t act, flags;
  uint32_t kpad;            // packed K (conv) / row pitch (fc), in elements
  uint32_t tiles_m, tiles_n;// tcgen05 conv: tile grid
  uint32_t ksplit;          // split-K factor (1 = none)
  uint32_t a_rows;          // tcgen05 conv: weight rows fetched per stage (TMA box), <= 128
  float* ws;                // split-K: fp32 partial sums, 64 x 128 per output tile, all zero between uses
  uint64_t* trace;          // debug (LF_TRACE): per-CTA phase timestamps
  const void* bmap;         // LF_TMA_B: device address of this slot's im2col CUtensorMap (128 B)
};

}  // namespace paella
