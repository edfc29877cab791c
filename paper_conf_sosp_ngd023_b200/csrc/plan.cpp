// Model planner: graph -> kernel chain, NHWC buffer plan, packed parameters.
//
// Paper: a job is the ordered sequence of its model's kernels (TVM's graph executor
// runs ops in order on one stream; §4.2 P943-951 waitlists follow stream semantics).
// Each kernel's static resource demand is known before launch (§4.1 P814-830:
// grid, block, shared memory, registers) -- the planner fixes grid/block/smem here
// and the CUDA backend reads registers from the compiled function.
//
//  * one kernel per non-concat node, plus the ingest (fp32 NCHW client input ->
//    NHWC, channels padded to 8) -- BN/ReLU/residual add are fused into the conv,
//    DenseNet's pre-activation BN+ReLU into the consuming conv/GAP as a prologue;
//  * concat = producers write disjoint channel ranges of one buffer (zero-copy);
//  * conv: groups==1 -> tcgen05 implicit GEMM (bf16) or SIMT implicit GEMM (fp32);
//    depthwise -> K2c;  FC -> GEMV;  pools / GAP -> SIMT.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <stdexcept>
#include <string>

#include "engine.h"

namespace paella {

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

static uint16_t f32_to_bf16_exact(float f, bool* exact) {
  uint32_t u;
  std::memcpy(&u, &f, 4);
  // RNE (inputs are required to be bf16-representable; flag otherwise)
  uint32_t r = (u + 0x7FFFu + ((u >> 16) & 1u)) >> 16;
  if ((u & 0xFFFFu) != 0) *exact = false;
  return (uint16_t)r;
}

struct Blob {
  std::vector<uint8_t>& b;
  size_t put(const void* p, size_t n) {
    size_t off = align_up(b.size(), 256);
    b.resize(off + n);
    if (p) std::memcpy(b.data() + off, p, n);
    return off;
  }
};

static bool use_tc() {
  const char* e = std::getenv("PAELLA_CONV");
  return !(e && std::string(e) == "simt");
}

uint32_t tc_tmem_cols() { return (TC_BN < 32 ? 32 : TC_BN) * TC_ACCS; }

int plan_model(Paella* P, const paella_model_desc_t* d, Model* m) {
  const uint32_t n = d->n_nodes;
  if (n < 2 || !d->nodes || d->nodes[0].op != PAELLA_OP_INPUT) return -EINVAL;
  if (d->dtype != PAELLA_DTYPE_BF16 && d->dtype != PAELLA_DTYPE_FP32) return -EINVAL;
  const size_t es = d->dtype == PAELLA_DTYPE_BF16 ? 2 : 4;
  m->name = d->name;
  m->dtype = d->dtype;
  m->nodes.assign(d->nodes, d->nodes + n);
  m->node_inputs.resize(n);
  for (uint32_t i = 0; i < n; ++i) {
    const paella_node_t& nd = d->nodes[i];
    for (uint32_t k = 0; k < nd.n_inputs; ++k) {
      int32_t s = nd.inputs[k];
      if (s < 0 || (uint32_t)s >= i) return -EINVAL;
      m->node_inputs[i].push_back(s);
    }
    if (nd.op != PAELLA_OP_INPUT && nd.n_inputs == 0) return -EINVAL;
    if (nd.op != PAELLA_OP_CONCAT && nd.op != PAELLA_OP_INPUT && nd.n_inputs != 1) return -EINVAL;
    if (nd.residual >= (int32_t)i) return -EINVAL;
    if (nd.op != PAELLA_OP_INPUT && nd.c % 8 != 0 && !(i == n - 1)) return -EINVAL;
  }
  const paella_node_t& in = d->nodes[0];
  if (in.c > 8) return -EINVAL;
  m->in_c = in.c;
  m->in_h = in.h;
  m->in_w = in.w;
  m->input_bytes = (size_t)in.c * in.h * in.w * 4;
  const paella_node_t& last = d->nodes[n - 1];
  if (last.op != PAELLA_OP_FC && last.op != PAELLA_OP_GAP) return -EINVAL;
  m->out_n = last.c;
  m->output_bytes = (size_t)last.c * 4;
  if (last.c % 8 != 0 && last.op == PAELLA_OP_GAP) return -EINVAL;

  // ---- buffer plan: concat aliasing, processed from the last node backwards ----
  m->buf_of.assign(n, -1);
  m->coff.assign(n, 0);
  auto new_buf = [&](uint32_t c, uint32_t h, uint32_t w) {
    m->bufs.push_back(Buffer{c, h, w, 0, 0});
    return (int32_t)m->bufs.size() - 1;
  };
  for (int32_t i = (int32_t)n - 1; i >= 0; --i) {
    const paella_node_t& nd = d->nodes[i];
    if (nd.op != PAELLA_OP_CONCAT) continue;
    if (m->buf_of[i] < 0) {
      int32_t first = m->node_inputs[i][0];
      if (m->buf_of[first] >= 0) {
        // a prefix of a later concat (DenseNet: every layer's input is a prefix of
        // the block's concat buffer): alias it
        m->buf_of[i] = m->buf_of[first];
        m->coff[i] = m->coff[first];
      } else {
        m->buf_of[i] = new_buf(nd.c, nd.h, nd.w);
        m->coff[i] = 0;
      }
    }
    uint32_t off = m->coff[i];
    for (int32_t s : m->node_inputs[i]) {
      const paella_node_t& sn = d->nodes[s];
      if (sn.op == PAELLA_OP_INPUT) return -EINVAL;
      if (m->buf_of[s] < 0) {
        m->buf_of[s] = m->buf_of[i];
        m->coff[s] = off;
      } else if (m->buf_of[s] != m->buf_of[i] || m->coff[s] != off) {
        return -EINVAL;   // a tensor in two non-prefix concats: unsupported layout
      }
      off += sn.c;
    }
    if (off != m->coff[i] + nd.c) return -EINVAL;
  }
  for (uint32_t i = 0; i < n; ++i) {
    const paella_node_t& nd = d->nodes[i];
    if (m->buf_of[i] >= 0) continue;
    if (i == n - 1) continue;                     // final output goes to client memory
    if (nd.op == PAELLA_OP_INPUT)
      m->buf_of[i] = new_buf(8, nd.h, nd.w);      // ingest pads channels to 8
    else
      m->buf_of[i] = new_buf(nd.c, nd.h, nd.w);
  }
  size_t ws = 0;
  for (auto& b : m->bufs) {
    b.bytes = (size_t)b.c * b.h * b.w * es;
    b.off = ws;
    ws = align_up(ws + b.bytes, 256);
  }
  m->slot_bytes = std::max<size_t>(ws, 256);

  // ---- kernels + packed parameters ----
  Blob blob{m->blob};
  const bool tc = use_tc() && d->dtype == PAELLA_DTYPE_BF16;
  bool exact = true;
  auto cs_of = [&](int32_t node) { return m->bufs[m->buf_of[node]].c; };

  {  // ingest
    KernelInst k;
    k.kind = KIND_INGEST;
    k.node = 0;
    k.out_buf = m->buf_of[0];
    LayerArgs& a = k.proto;
    a.cin = in.c;
    a.h = in.h;
    a.w_ = in.w;
    a.cout = 8;
    a.oh = in.h;
    a.ow = in.w;
    a.out_cs = 8;
    a.out_co = 0;
    // the input streams over PCIe from client memory: the read latency (~1-2 us per
    // request) is covered by requests in flight, so the 4-pixel path runs 64-thread
    // blocks to spread over >= the 148 SMs (224 x 224: 196 CTAs instead of 49)
    const bool quad = in.h * in.w % 4 == 0;
    k.block = quad ? 64 : 256;
    k.grid[0] = quad ? (in.h * in.w / 4 + k.block - 1) / k.block : (in.h * in.w + 255) / 256;
    k.bytes = (uint64_t)in.c * in.h * in.w * 4 + (uint64_t)8 * in.h * in.w * es;
    m->kernels.push_back(k);
  }

  // GAP whose only consumer is an FC: fused into one gap_fc kernel
  std::vector<uint32_t> consumers(n, 0);
  for (uint32_t i = 0; i < n; ++i) {
    for (int32_t s : m->node_inputs[i]) consumers[s]++;
    if (d->nodes[i].residual >= 0) consumers[d->nodes[i].residual]++;
  }
  std::vector<bool> fused_gap(n, false);
  const bool fuse = !std::getenv("PAELLA_NO_FUSE");
  for (uint32_t i = 1; i < n; ++i) {
    const paella_node_t& nd = d->nodes[i];
    if (fuse && nd.op == PAELLA_OP_FC) {
      int32_t src = m->node_inputs[i][0];
      const paella_node_t& sn = d->nodes[src];
      if (sn.op == PAELLA_OP_GAP && consumers[src] == 1 && sn.c % 8 == 0 && sn.c <= 8192) fused_gap[src] = true;
    }
  }
  for (uint32_t i = 1; i < n; ++i) {
    const paella_node_t& nd = d->nodes[i];
    if (nd.op == PAELLA_OP_CONCAT || fused_gap[i]) continue;
    int32_t src = m->node_inputs[i][0];
    const paella_node_t& sn = d->nodes[src];
    const bool is_first = sn.op == PAELLA_OP_INPUT;
    const uint32_t cin = is_first ? 8 : sn.c;   // channels the kernel reads
    KernelInst k;
    k.node = (int32_t)i;
    k.in_buf = m->buf_of[src];
    k.out_buf = (i == n - 1) ? -1 : m->buf_of[i];
    LayerArgs& a = k.proto;
    a.in_cs = cs_of(src);
    a.in_co = m->coff[src];
    if (k.out_buf >= 0) {
      a.out_cs = cs_of(i);
      a.out_co = m->coff[i];
    }
    a.cin = cin;
    a.h = sn.h;
    a.w_ = sn.w;
    a.cout = nd.c;
    a.oh = nd.h;
    a.ow = nd.w;
    a.kh = nd.kh;
    a.kw = nd.kw;
    a.sh = nd.sh;
    a.sw = nd.sw;
    a.ph = nd.ph;
    a.pw = nd.pw;
    a.groups = nd.groups ? nd.groups : 1;
    a.act = nd.act;
    a.ksplit = 1;
    a.a_rows = TC_BM;
    if (i == n - 1) a.flags |= LF_FINAL;
    if (nd.flags & PAELLA_NODE_PROLOGUE) {
      if (!nd.pro_scale || !nd.pro_shift) return -EINVAL;
      a.flags |= LF_PROLOGUE;
      k.has_pro = true;
      k.ps_off = blob.put(nd.pro_scale, sn.c * 4);
      k.pz_off = blob.put(nd.pro_shift, sn.c * 4);
    }
    if (nd.residual >= 0) {
      if (nd.op != PAELLA_OP_CONV) return -EINVAL;
      a.flags |= LF_RESIDUAL;
      k.res_buf = m->buf_of[nd.residual];
      a.res_cs = cs_of(nd.residual);
      a.res_co = m->coff[nd.residual];
    }
    const uint32_t P_out = nd.h * nd.w;
    switch (nd.op) {
      case PAELLA_OP_CONV: {
        const uint32_t g = a.groups;
        const uint32_t cin_real = sn.c;
        if (!nd.weight) return -EINVAL;
        std::vector<float> bias(nd.c, 0.f);
        if (nd.bias) std::memcpy(bias.data(), nd.bias, nd.c * 4);
        k.b_off = blob.put(bias.data(), nd.c * 4);
        if (g == 1) {
          const uint32_t K = nd.kh * nd.kw * cin;
          const uint32_t kpad = (uint32_t)align_up(K, 64);
          a.kpad = kpad;
          const bool use_tc_here = tc;
          const uint32_t rows = use_tc_here ? (uint32_t)align_up(nd.c, TC_BM) : nd.c;
          // pack [rows][kpad], k = (r, s, ci)
          std::vector<float> wp((size_t)rows * kpad, 0.f);
          for (uint32_t co = 0; co < nd.c; ++co)
            for (uint32_t r = 0; r < nd.kh; ++r)
              for (uint32_t s = 0; s < nd.kw; ++s)
                for (uint32_t ci = 0; ci < cin_real; ++ci)
                  wp[(size_t)co * kpad + (r * nd.kw + s) * cin + ci] =
                      nd.weight[(((size_t)co * cin_real + ci) * nd.kh + r) * nd.kw + s];
          if (es == 2) {
            std::vector<uint16_t> wb(wp.size());
            for (size_t q = 0; q < wp.size(); ++q) wb[q] = f32_to_bf16_exact(wp[q], &exact);
            k.w_off = blob.put(wb.data(), wb.size() * 2);
            k.w_bytes = wb.size() * 2;
          } else {
            k.w_off = blob.put(wp.data(), wp.size() * 4);
            k.w_bytes = wp.size() * 4;
          }
          if (use_tc_here) {
            k.kind = (a.flags & LF_PROLOGUE) ? KIND_CONV_TC_PRO : KIND_CONV_TC;
            a.tiles_m = rows / TC_BM;
            a.tiles_n = (P_out + TC_BN - 1) / TC_BN;
            uint32_t nk = kpad / TC_BK;
            uint32_t tiles = a.tiles_m * a.tiles_n;
            // split K so the grid approaches one wave of SMs, >= 2 k-blocks per split;
            // the splits of a tile form one thread-block cluster
            uint32_t split = 1;
            const char* e = std::getenv("PAELLA_NOSPLIT");
            if (!e) {
              // splitting pays only for deep K: a cluster barrier + DSMEM reduction cost ~1 us;
              // clusters of up to 16 CTAs (non-portable size, allowed on sm_100)
              // measured (kernel_times): with the restricted-fence cluster barrier and the
              // staggered DSMEM reduction, splits down to 2 k-blocks each pay from nk >= 6
              static const uint32_t min_nk = std::getenv("PAELLA_SPLIT_MIN_NK") ? atoi(std::getenv("PAELLA_SPLIT_MIN_NK")) : 6;
              static const uint32_t min_st = std::getenv("PAELLA_SPLIT_MIN_STAGES") ? atoi(std::getenv("PAELLA_SPLIT_MIN_STAGES")) : 2;
              if (nk >= min_nk)
                while (split < 16 && tiles * split * 2 <= P->sms && nk / (split * 2) >= min_st) split *= 2;
            }
            a.ksplit = split;
            if (std::getenv("PAELLA_SPLIT_DSMEM")) a.flags |= LF_SPLIT_DSMEM;   // A/B: the DSMEM reduction
            if (std::getenv("PAELLA_SPLIT_NOROT")) a.flags |= LF_SPLIT_NOROT;
            if (std::getenv("PAELLA_SPLIT_RELBAR")) a.flags |= LF_SPLIT_RELBAR;
            if (std::getenv("PAELLA_MBAR_SPIN")) a.flags |= LF_MBAR_SPIN;
            // narrow layers: fetch only the live weight rows (SW128 atoms are 8 rows)
            a.a_rows = nd.c < TC_BM ? (uint32_t)align_up(nd.c, 8) : TC_BM;
            k.tmem_cols = tc_tmem_cols();
            // saturating shapes (>= 2 waves of 64-pixel tiles at 2 CTAs/SM, no split, no
            // prologue): 128-pixel tiles halve the weight traffic per flop.  Batch-1
            // serving layers stay below this (at most 196 tiles of 64 pixels at 224^2).
            if (k.kind == KIND_CONV_TC && split == 1 && tiles >= 4 * P->sms && !std::getenv("PAELLA_NO_WIDE")) {
              k.kind = KIND_CONV_TC128;
              a.tiles_n = (P_out + TC_BN_WIDE - 1) / TC_BN_WIDE;
              k.tmem_cols = TC_BN_WIDE * TC_ACCS;
            }
            // narrow layers (<= 64 output channels, no prologue): UMMA M = 64, so the tensor
            // core reads 64 weight rows per k-block instead of 128 (half of them zero)
            // Opt-in (PAELLA_M64): faster in isolation (DenseNet-121 -3.7 %) but the C-3 mix's
            // device-only saturation rate drops ~5 % (profiles/r2/diag/split_gain)
            if (k.kind == KIND_CONV_TC && a.a_rows <= 64 && std::getenv("PAELLA_M64")) k.kind = KIND_CONV_TC_M64;
            // activations by TMA im2col: one 64-channel slice of one filter tap per k-block
            // (cin % 64 == 0), 16-byte aligned pixel rows, no in-place prologue
            if (k.kind != KIND_CONV_TC_PRO && a.cin % 64 == 0 && a.in_cs % 8 == 0 && a.in_co % 8 == 0 &&
                a.sh <= 8 && a.sw <= 8 && a.ph < 128 && a.pw < 128 && a.kh <= 128 && a.kw <= 128 &&
                !std::getenv("PAELLA_NO_TMA_B"))
              a.flags |= LF_TMA_B;
            k.grid[0] = a.tiles_n;
            k.grid[1] = a.tiles_m;
            k.grid[2] = split;
            k.block = TC_THREADS;
            k.smem = tc_smem_bytes();

          } else {
            k.kind = KIND_CONV_SIMT;
            k.grid[0] = (P_out + 63) / 64;
            k.grid[1] = (nd.c + 63) / 64;
            k.block = 256;
          }
          k.flops = 2ull * nd.c * P_out * nd.kh * nd.kw * cin_real;
          k.bytes = (uint64_t)nd.c * nd.kh * nd.kw * cin_real * es + (uint64_t)sn.h * sn.w * cin_real * es +
                    (uint64_t)P_out * nd.c * es * ((a.flags & LF_RESIDUAL) ? 2 : 1);
        } else if (g == cin_real && g == nd.c) {
          // depthwise: pack [kh][kw][c]
          std::vector<float> wp((size_t)nd.kh * nd.kw * nd.c);
          for (uint32_t c = 0; c < nd.c; ++c)
            for (uint32_t r = 0; r < nd.kh; ++r)
              for (uint32_t s = 0; s < nd.kw; ++s)
                wp[((size_t)r * nd.kw + s) * nd.c + c] = nd.weight[((size_t)c * nd.kh + r) * nd.kw + s];
          if (es == 2) {
            std::vector<uint16_t> wb(wp.size());
            for (size_t q = 0; q < wp.size(); ++q) wb[q] = f32_to_bf16_exact(wp[q], &exact);
            k.w_off = blob.put(wb.data(), wb.size() * 2);
          } else {
            k.w_off = blob.put(wp.data(), wp.size() * 4);
          }
          k.kind = KIND_DWCONV;
          k.grid[0] = (P_out * (nd.c / 8) + 255) / 256;
          k.block = 256;
          k.flops = 2ull * nd.c * P_out * nd.kh * nd.kw;
          k.bytes = (uint64_t)nd.c * nd.kh * nd.kw * es + (uint64_t)sn.h * sn.w * nd.c * es +
                    (uint64_t)P_out * nd.c * es * ((a.flags & LF_RESIDUAL) ? 2 : 1);
        } else {
          return -EINVAL;   // grouped conv other than depthwise: not in the model mix
        }
        break;
      }
      case PAELLA_OP_MAXPOOL:
      case PAELLA_OP_AVGPOOL: {
        k.kind = nd.op == PAELLA_OP_MAXPOOL ? KIND_MAXPOOL : KIND_AVGPOOL;
        if (nd.flags & PAELLA_NODE_CEIL) a.flags |= LF_CEIL;
        if (nd.c != sn.c) return -EINVAL;
        k.grid[0] = (P_out * (nd.c / 8) + 255) / 256;
        k.block = 256;
        k.bytes = (uint64_t)sn.h * sn.w * sn.c * es + (uint64_t)P_out * nd.c * es;
        break;
      }
      case PAELLA_OP_SPIN: {   // Fig. 2 synthetic kernel (HoL microbenchmark)
        k.kind = KIND_SPIN;
        if (nd.c != cin || nd.h != sn.h || nd.w != sn.w || nd.h * nd.w != 1 || nd.c % 8) return -EINVAL;
        k.grid[0] = 1;
        k.block = 128;
        k.bytes = 2ull * nd.c * es;
        break;
      }
      case PAELLA_OP_GAP: {
        k.kind = KIND_GAP;
        if (nd.c != sn.c || sn.c % 8) return -EINVAL;
        k.grid[0] = (nd.c / 8 * 32 + 255) / 256;   // a warp per 8-channel granule
        k.block = 256;
        k.bytes = (uint64_t)sn.h * sn.w * sn.c * es + (uint64_t)nd.c * ((a.flags & LF_FINAL) ? 4 : es);
        break;
      }
      case PAELLA_OP_FC: {
        if (fused_gap[src]) {
          // read the GAP's input (C x H x W) directly, with the GAP's prologue
          const paella_node_t& gn = sn;
          int32_t gsrc = m->node_inputs[src][0];
          const paella_node_t& gin = d->nodes[gsrc];
          k.kind = KIND_GAPFC;
          k.in_buf = m->buf_of[gsrc];
          a.in_cs = cs_of(gsrc);
          a.in_co = m->coff[gsrc];
          a.cin = gn.c;
          a.h = gin.h;
          a.w_ = gin.w;
          a.kpad = gn.c;
          if (gn.flags & PAELLA_NODE_PROLOGUE) {
            if (!gn.pro_scale || !gn.pro_shift) return -EINVAL;
            a.flags |= LF_PROLOGUE;
            k.has_pro = true;
            k.ps_off = blob.put(gn.pro_scale, gn.c * 4);
            k.pz_off = blob.put(gn.pro_shift, gn.c * 4);
          }
          std::vector<float> wp(nd.weight, nd.weight + (size_t)nd.c * gn.c);
          if (es == 2) {
            std::vector<uint16_t> wb(wp.size());
            for (size_t q = 0; q < wp.size(); ++q) wb[q] = f32_to_bf16_exact(wp[q], &exact);
            k.w_off = blob.put(wb.data(), wb.size() * 2);
          } else {
            k.w_off = blob.put(wp.data(), wp.size() * 4);
          }
          std::vector<float> bias(nd.c, 0.f);
          if (nd.bias) std::memcpy(bias.data(), nd.bias, nd.c * 4);
          k.b_off = blob.put(bias.data(), nd.c * 4);
          // one FC row per warp, 8 warps per CTA, whole clusters of GAPFC_CLUSTER CTAs
          k.grid[0] = ((nd.c + 7) / 8 + GAPFC_CLUSTER - 1) / GAPFC_CLUSTER * GAPFC_CLUSTER;
          k.block = 256;
          k.smem = gn.c * 4;
          k.flops = 2ull * nd.c * gn.c + (uint64_t)gn.c * gin.h * gin.w;
          k.bytes = (uint64_t)nd.c * gn.c * es + (uint64_t)gin.h * gin.w * gn.c * es +
                    (uint64_t)nd.c * ((a.flags & LF_FINAL) ? 4 : es);
          break;
        }
        k.kind = KIND_FC;
        const uint32_t K = sn.c * sn.h * sn.w;
        if (K % 8 || (sn.h * sn.w > 1 && a.in_cs != sn.c)) return -EINVAL;
        if (!nd.weight) return -EINVAL;
        a.cin = K;
        a.kpad = K;
        // torch flattens NCHW (c*HW + p); our activation is NHWC (p*C + c)
        const uint32_t HW = sn.h * sn.w, C = sn.c;
        std::vector<float> wp((size_t)nd.c * K);
        for (uint32_t o = 0; o < nd.c; ++o)
          for (uint32_t c = 0; c < C; ++c)
            for (uint32_t p = 0; p < HW; ++p)
              wp[(size_t)o * K + (size_t)p * C + c] = nd.weight[(size_t)o * K + (size_t)c * HW + p];
        if (es == 2) {
          std::vector<uint16_t> wb(wp.size());
          for (size_t q = 0; q < wp.size(); ++q) wb[q] = f32_to_bf16_exact(wp[q], &exact);
          k.w_off = blob.put(wb.data(), wb.size() * 2);
        } else {
          k.w_off = blob.put(wp.data(), wp.size() * 4);
        }
        std::vector<float> bias(nd.c, 0.f);
        if (nd.bias) std::memcpy(bias.data(), nd.bias, nd.c * 4);
        k.b_off = blob.put(bias.data(), nd.c * 4);
        k.grid[0] = (nd.c + 7) / 8;
        k.block = 256;
        k.flops = 2ull * nd.c * K;
        k.bytes = (uint64_t)nd.c * K * es + (uint64_t)K * es + (uint64_t)nd.c * ((a.flags & LF_FINAL) ? 4 : es);
        break;
      }
      default:
        return -EINVAL;
    }
    m->kernels.push_back(k);
  }
  if (!exact && es == 2) return -EINVAL;   // bf16 path requires bf16-representable weights

  // ---- NEXT-4: the kernel DAG and its virtual streams (Fig. 7 waitlists) ----
  // producers(node) = the kernels that write node's tensor: its own kernel, or through a
  // concat (no kernel, zero-copy) the producers of its inputs, or through a GAP fused
  // into its FC the producers of the GAP's input
  std::vector<int32_t> kernel_of(n, -1);
  for (uint32_t k = 0; k < m->kernels.size(); ++k) kernel_of[m->kernels[k].node < 0 ? 0 : m->kernels[k].node] = k;
  kernel_of[0] = 0;
  std::vector<std::vector<uint32_t>> prod(n);
  for (uint32_t i = 0; i < n; ++i) {
    if (kernel_of[i] >= 0 && !fused_gap[i]) {
      prod[i] = {(uint32_t)kernel_of[i]};
    } else {
      for (int32_t s : m->node_inputs[i]) prod[i].insert(prod[i].end(), prod[s].begin(), prod[s].end());
    }
  }
  const uint32_t nk = (uint32_t)m->kernels.size();
  std::vector<int32_t> tail_of_vs;   // last kernel of each virtual stream so far
  for (uint32_t k = 0; k < nk; ++k) {
    KernelInst& K = m->kernels[k];
    std::vector<uint32_t> deps;
    if (k > 0) {
      const uint32_t node = (uint32_t)K.node;
      for (int32_t s : m->node_inputs[node]) deps.insert(deps.end(), prod[s].begin(), prod[s].end());
      if (d->nodes[node].residual >= 0) {
        const auto& r = prod[d->nodes[node].residual];
        deps.insert(deps.end(), r.begin(), r.end());
      }
    }
    std::sort(deps.begin(), deps.end());
    deps.erase(std::unique(deps.begin(), deps.end()), deps.end());
    for (uint32_t x : deps)
      if (x >= k) return -EINVAL;
    K.deps = deps;
    // virtual stream: continue the stream whose tail is the most recent dependency;
    // otherwise open a new one (at most MAX_VS), else join the latest dependency's
    int32_t vs = -1;
    for (auto it = deps.rbegin(); it != deps.rend() && vs < 0; ++it)
      if (tail_of_vs[m->kernels[*it].vs] == (int32_t)*it) vs = (int32_t)m->kernels[*it].vs;
    if (vs < 0) {
      if (tail_of_vs.size() < MAX_VS || deps.empty()) {
        vs = deps.empty() && !tail_of_vs.empty() ? 0 : (int32_t)tail_of_vs.size();
        if (vs == (int32_t)tail_of_vs.size()) tail_of_vs.push_back(-1);
      } else {
        vs = (int32_t)m->kernels[deps.back()].vs;
      }
    }
    K.vs = (uint32_t)vs;
    tail_of_vs[vs] = (int32_t)k;
  }
  m->n_vs = (uint32_t)tail_of_vs.size();
  for (uint32_t k = 0; k < nk; ++k)
    for (uint32_t x : m->kernels[k].deps)
      if (m->kernels[x].vs != m->kernels[k].vs) m->kernels[x].xout = true;
  return 0;
}

}  // namespace paella
