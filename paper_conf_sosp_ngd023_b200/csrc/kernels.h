// Kernel kinds of the CUDA path and their launch table.
#pragma once
#include <stdint.h>

namespace paella {

enum KernelKind : uint32_t {
  KIND_INGEST = 0,
  KIND_CONV_SIMT = 1,
  KIND_CONV_TC = 2,     // tcgen05 implicit-GEMM conv (bf16)
  KIND_DWCONV = 3,
  KIND_MAXPOOL = 4,
  KIND_AVGPOOL = 5,
  KIND_GAP = 6,
  KIND_FC = 7,
  KIND_EMPTY = 8,
  KIND_CONV_TC_PRO = 9, // tcgen05 conv with the per-channel affine+ReLU input prologue
  KIND_GAPFC = 10,      // fused global average pool + FC classifier head
  KIND_SPIN = 11,       // synthetic HoL-microbenchmark kernel (Fig. 2): one resident block
  KIND_CONV_TC128 = 12, // tcgen05 conv with 128-pixel tiles (saturating shapes, no split-K)
  KIND_CONV_TC_M64 = 13,  // tcgen05 conv with UMMA M = 64 (layers with <= 64 output channels)
  KIND_COUNT = 14,
};

typedef void (*KernelFn)();

void simt_kernel_table(KernelFn (&bf16_instr)[KIND_COUNT], KernelFn (&bf16_plain)[KIND_COUNT],
                       KernelFn (&f32_instr)[KIND_COUNT], KernelFn (&f32_plain)[KIND_COUNT]);

KernelFn gate_kernel();   // k_gate(const volatile uint32_t* flag)
KernelFn clock_kernel();  // k_clock_probe(flag, out, n): globaltimer ping-pong
KernelFn mirror_kernel();  // k_notify_mirror(ctrs, host_mirror, state)
KernelFn proxy_kernel();  // k_notify_proxy(dev_ring, host_ring, mask, log2cap, state)

// tcgen05 conv: instrumented / plain instantiations [0] plain input, [1] prologue
void tc_kernel_table(KernelFn* instr, KernelFn* plain);
constexpr uint32_t TC_BM = 128;       // Cout rows per CTA (UMMA M, TMEM lanes)
constexpr uint32_t TC_BN = 64;        // output pixels per CTA (UMMA N)
constexpr uint32_t TC_BK = 64;        // K per pipeline stage (128 B of bf16 = one swizzle row)
#ifndef PAELLA_TC_STAGES
#define PAELLA_TC_STAGES 4   // (A/B build variant: build.py PAELLA_DEFINES=-DPAELLA_TC_STAGES=8)
#endif
constexpr uint32_t TC_STAGES = PAELLA_TC_STAGES;
#ifndef PAELLA_TC_ACCS
#define PAELLA_TC_ACCS 1     // (A/B build variant) TMEM accumulators alternated over k-blocks
#endif
constexpr uint32_t TC_ACCS = PAELLA_TC_ACCS;
constexpr uint32_t TC_RING = TC_STAGES * (TC_BM * TC_BK * 2 + TC_BN * TC_BK * 2);   // 96 KiB stage ring
constexpr uint32_t TC_BN_WIDE = 128;   // KIND_CONV_TC128: 3 stages of 16 + 16 KiB in the same ring
constexpr uint32_t GAPFC_CLUSTER = 8;   // fused GAP+FC head: CTAs per cluster (pooling split)
constexpr uint32_t TC_THREADS = 192;    // 4 producer/epilogue warps + 1 MMA warp + 1 bookkeeping warp
uint32_t tc_smem_bytes();

}  // namespace paella
