// bvh.cpp -- sr_scene_build: binned-SAH BVH over a triangle soup, written as
// the device scene image of pt_scene.h (config 4).  Host code, single
// threaded, deterministic for a given input.
//
// The BVH is an acceleration structure only: the pathtrace kernels must
// return exactly the brute-force closest hit (reading R7), so every
// child box is padded outward and the kernels' slab test is conservative.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>
#include <string>
#include <vector>

#include "pt_scene.h"
#include "sr_internal.h"

namespace sr {
namespace {

constexpr int kBins = 16;
constexpr int kLeafMax = 8;   // a leaf never holds more than this many triangles
constexpr int kLeafMin = 2;   // ranges this small always become leaves

struct Box {
  float lo[3] = {INFINITY, INFINITY, INFINITY};
  float hi[3] = {-INFINITY, -INFINITY, -INFINITY};
  void grow(const Box& b) {
    for (int k = 0; k < 3; ++k) {
      lo[k] = std::min(lo[k], b.lo[k]);
      hi[k] = std::max(hi[k], b.hi[k]);
    }
  }
  void grow(const float* p) {
    for (int k = 0; k < 3; ++k) {
      lo[k] = std::min(lo[k], p[k]);
      hi[k] = std::max(hi[k], p[k]);
    }
  }
  double area() const {
    if (!(hi[0] >= lo[0])) return 0.0;
    const double dx = hi[0] - lo[0], dy = hi[1] - lo[1], dz = hi[2] - lo[2];
    return 2.0 * (dx * dy + dy * dz + dz * dx);
  }
};

struct BNode {
  Box box;
  int left = -1, right = -1;  // build-node children (inner)
  int start = 0, count = 0;   // leaf range (count > 0)
};

struct Job {
  int node, start, end;
};

struct Builder {
  const float* tris;
  std::vector<Box> pbox;
  std::vector<float> cen;  // 3 per primitive
  std::vector<uint32_t> idx;
  std::vector<BNode> nodes;

  int make_leaf(int n, int start, int count) {
    nodes[n].start = start;
    nodes[n].count = count;
    return n;
  }

  void build() {
    const size_t n = pbox.size();
    idx.resize(n);
    for (size_t i = 0; i < n; ++i) idx[i] = (uint32_t)i;
    nodes.reserve(2 * n + 1);
    nodes.emplace_back();
    std::vector<Job> stack{{0, 0, (int)n}};
    while (!stack.empty()) {
      const Job j = stack.back();
      stack.pop_back();
      Box box, cb;
      for (int i = j.start; i < j.end; ++i) {
        box.grow(pbox[idx[i]]);
        cb.grow(&cen[3 * (size_t)idx[i]]);
      }
      nodes[j.node].box = box;
      const int count = j.end - j.start;
      if (count <= kLeafMin) { make_leaf(j.node, j.start, count); continue; }
      int axis = 0;
      float ext = cb.hi[0] - cb.lo[0];
      for (int k = 1; k < 3; ++k)
        if (cb.hi[k] - cb.lo[k] > ext) { ext = cb.hi[k] - cb.lo[k]; axis = k; }
      int split = -1;
      if (ext > 0.0f) {
        Box bb[kBins];
        int bc[kBins] = {0};
        const double scale = kBins / (double)ext;
        auto bin_of = [&](uint32_t p) {
          const int b = (int)((cen[3 * (size_t)p + axis] - cb.lo[axis]) * scale);
          return std::min(std::max(b, 0), kBins - 1);
        };
        for (int i = j.start; i < j.end; ++i) {
          const int b = bin_of(idx[i]);
          bb[b].grow(pbox[idx[i]]);
          bc[b]++;
        }
        double rightA[kBins];
        int rightN[kBins];
        Box acc;
        int an = 0;
        for (int b = kBins - 1; b > 0; --b) {
          acc.grow(bb[b]);
          an += bc[b];
          rightA[b] = acc.area();
          rightN[b] = an;
        }
        Box lacc;
        int ln = 0;
        double best = INFINITY;
        for (int b = 1; b < kBins; ++b) {
          lacc.grow(bb[b - 1]);
          ln += bc[b - 1];
          if (ln == 0 || rightN[b] == 0) continue;
          const double cost = lacc.area() * ln + rightA[b] * rightN[b];
          if (cost < best) { best = cost; split = b; }
        }
        const double leaf_cost = (double)count;
        const double split_cost = 1.0 + best / std::max(box.area(), 1e-30);
        if (split >= 0 && count <= kLeafMax && split_cost >= leaf_cost) split = -1;
        if (split >= 0) {
          auto mid = std::stable_partition(idx.begin() + j.start, idx.begin() + j.end,
                                           [&](uint32_t p) { return bin_of(p) < split; });
          const int m = (int)(mid - idx.begin());
          if (m == j.start || m == j.end) split = -1;
          else { push_children(j, m, stack); continue; }
        }
      }
      if (count <= kLeafMax) { make_leaf(j.node, j.start, count); continue; }
      // degenerate centroids: split the range in half in a stable order
      std::stable_sort(idx.begin() + j.start, idx.begin() + j.end,
                       [&](uint32_t a, uint32_t b) {
                         return cen[3 * (size_t)a + axis] < cen[3 * (size_t)b + axis];
                       });
      push_children(j, j.start + count / 2, stack);
    }
  }

  void push_children(const Job& j, int m, std::vector<Job>& stack) {
    const int l = (int)nodes.size();
    nodes.emplace_back();
    nodes.emplace_back();
    nodes[j.node].left = l;
    nodes[j.node].right = l + 1;
    stack.push_back({l + 1, m, j.end});
    stack.push_back({l, j.start, m});
  }
};

float pad_lo(float v) { return std::nextafter(v - std::fabs(v) * 1e-5f - 1e-6f, -INFINITY); }
float pad_hi(float v) { return std::nextafter(v + std::fabs(v) * 1e-5f + 1e-6f, INFINITY); }

size_t image_bound(uint32_t n_tris, uint32_t n_mats) {
  const size_t nodes = std::max<size_t>(n_tris, 1);
  return sizeof(PtHeader) + nodes * sizeof(PtNode) + (size_t)n_tris * sizeof(PtTri) +
         (size_t)n_mats * sizeof(PtMat);
}

}  // namespace

std::string check_scene_inputs(const float* tris, const uint32_t* mat, uint32_t n_tris,
                               const float* mats, uint32_t n_mats, const float* cam) {
  if (n_tris == 0) return "n_tris must be >= 1";
  if (n_tris >= (1u << 31)) return "n_tris must be < 2^31 (BVH references are int32)";
  if (!tris || !mat || !mats || !cam) return "NULL input array";
  if (n_mats == 0) return "n_mats must be >= 1";
  for (size_t i = 0; i < 9 * (size_t)n_tris; ++i)
    if (!std::isfinite(tris[i])) return "non-finite vertex coordinate at triangle " +
                                        std::to_string(i / 9);
  for (uint32_t i = 0; i < n_tris; ++i)
    if (mat[i] >= n_mats) return "material id out of range at triangle " + std::to_string(i);
  for (uint32_t m = 0; m < n_mats; ++m) {
    const float k = mats[8 * (size_t)m];
    if (!(k == 0.0f || k == 1.0f || k == 2.0f || k == 3.0f))
      return "material kind must be 0..3";
  }
  return "";
}

}  // namespace sr

using namespace sr;

// Builds the scene image; copies it to dst with cudaMemcpy (device) or memcpy
// (host).  Shared by sr_scene_build and sr_scene_build_host.
static int build_scene(const char* fn, bool to_device, const float* tris, const uint32_t* mat,
                       uint32_t n_tris, const float* mats, uint32_t n_mats, const float* cam,
                       void* dst, size_t dst_bytes, size_t* needed) {
  if (needed) *needed = 0;
  const std::string why = check_scene_inputs(tris, mat, n_tris, mats, n_mats, cam);
  if (!why.empty()) return set_error(SR_E_INVALID, std::string(fn) + ": " + why);
  const size_t bound = image_bound(n_tris, n_mats);
  if (needed) *needed = bound;
  if (!dst) return SR_OK;
  if (dst_bytes < bound) return set_error(SR_E_NOMEM, std::string(fn) + ": dst_bytes < needed");

  Builder B;
  B.tris = tris;
  B.pbox.resize(n_tris);
  B.cen.resize(3 * (size_t)n_tris);
  for (uint32_t i = 0; i < n_tris; ++i) {
    const float* t = tris + 9 * (size_t)i;
    Box b;
    b.grow(t);
    b.grow(t + 3);
    b.grow(t + 6);
    B.pbox[i] = b;
    for (int k = 0; k < 3; ++k) B.cen[3 * (size_t)i + k] = 0.5f * (b.lo[k] + b.hi[k]);
  }
  B.build();

  // flatten: one PtNode per inner build node, pre-order; leaves fold into refs
  std::vector<int> out_of(B.nodes.size(), -1);
  std::vector<int> order;
  {
    std::vector<int> st{0};
    while (!st.empty()) {
      const int n = st.back();
      st.pop_back();
      if (B.nodes[n].count > 0 && n != 0) continue;
      out_of[n] = (int)order.size();
      order.push_back(n);
      if (B.nodes[n].count == 0) {
        st.push_back(B.nodes[n].right);
        st.push_back(B.nodes[n].left);
      }
    }
  }
  std::vector<PtNode> nodes(order.size());
  auto set_child = [&](PtNode& o, int slot, int c) {
    int32_t& ref = slot ? o.ref1 : o.ref0;
    int32_t& cnt = slot ? o.cnt1 : o.cnt0;
    if (c < 0) {
      for (int k = 0; k < 3; ++k) { o.lo[k][slot] = INFINITY; o.hi[k][slot] = -INFINITY; }
      ref = -1;
      cnt = 0;
      return;
    }
    const BNode& b = B.nodes[c];
    for (int k = 0; k < 3; ++k) {
      o.lo[k][slot] = pad_lo(b.box.lo[k]);
      o.hi[k][slot] = pad_hi(b.box.hi[k]);
    }
    if (b.count > 0) { ref = b.start; cnt = b.count; }
    else { ref = out_of[c]; cnt = 0; }
  };
  for (size_t i = 0; i < order.size(); ++i) {
    const BNode& b = B.nodes[order[i]];
    if (b.count > 0) {           // the root itself is a leaf: wrap it
      set_child(nodes[i], 0, order[i]);
      set_child(nodes[i], 1, -1);
    } else {
      set_child(nodes[i], 0, b.left);
      set_child(nodes[i], 1, b.right);
    }
  }

  // traversal stack bound: a visit pushes at most one entry (the farther of
  // two inner children), so a ray holds at most (inner nodes on its root path
  // - 1) entries
  uint32_t stack_need = 0;
  {
    std::vector<std::pair<int, uint32_t>> st{{0, 0u}};
    while (!st.empty()) {
      const auto [i, d] = st.back();
      st.pop_back();
      stack_need = std::max(stack_need, d);
      const PtNode& o = nodes[i];
      const bool in0 = o.ref0 >= 0 && o.cnt0 == 0, in1 = o.ref1 >= 0 && o.cnt1 == 0;
      const uint32_t dd = d + ((in0 && in1) ? 1u : 0u);
      if (in0) st.push_back({o.ref0, dd});
      if (in1) st.push_back({o.ref1, dd});
    }
  }

  std::vector<unsigned char> img(bound, 0);
  PtHeader h{};
  h.stack_need = stack_need;
  h.magic = kPtMagic;
  h.n_nodes = (uint32_t)nodes.size();
  h.n_tris = n_tris;
  h.n_mats = n_mats;
  h.off_nodes = sizeof(PtHeader);
  h.off_tris = h.off_nodes + nodes.size() * sizeof(PtNode);
  h.off_mats = h.off_tris + (size_t)n_tris * sizeof(PtTri);
  h.bytes = h.off_mats + (size_t)n_mats * sizeof(PtMat);
  std::memcpy(h.cam, cam, 14 * sizeof(float));
  std::memcpy(img.data(), &h, sizeof h);
  std::memcpy(img.data() + h.off_nodes, nodes.data(), nodes.size() * sizeof(PtNode));
  PtTri* T = reinterpret_cast<PtTri*>(img.data() + h.off_tris);
  for (uint32_t k = 0; k < n_tris; ++k) {
    const uint32_t i = B.idx[k];
    const float* t = tris + 9 * (size_t)i;
    PtTri& o = T[k];
    for (int c = 0; c < 3; ++c) {
      o.v0[c] = t[c];
      o.e1[c] = t[3 + c] - t[c];   // binary32 subtraction, as the oracle does
      o.e2[c] = t[6 + c] - t[c];
    }
    o.id = i;
    o.mat = mat[i];
    o.pad = 0;
  }
  std::memcpy(img.data() + h.off_mats, mats, (size_t)n_mats * sizeof(PtMat));
  if (to_device) {
    const cudaError_t e = cudaMemcpy(dst, img.data(), h.bytes, cudaMemcpyHostToDevice);
    if (e != cudaSuccess)
      return set_error(SR_E_CUDA, std::string(fn) + ": cudaMemcpy: " + cudaGetErrorString(e));
    register_scene(dst, &h);
  } else {
    std::memcpy(dst, img.data(), h.bytes);
  }
  if (needed) *needed = h.bytes;
  return SR_OK;
}

extern "C" int sr_scene_build(const float* tris, const uint32_t* mat, uint32_t n_tris,
                              const float* mats, uint32_t n_mats, const float* cam, void* dst_dev,
                              size_t dst_bytes, size_t* needed) {
  return build_scene("sr_scene_build", true, tris, mat, n_tris, mats, n_mats, cam, dst_dev,
                     dst_bytes, needed);
}

extern "C" int sr_scene_build_host(const float* tris, const uint32_t* mat, uint32_t n_tris,
                                   const float* mats, uint32_t n_mats, const float* cam,
                                   void* dst_host, size_t dst_bytes, size_t* needed) {
  return build_scene("sr_scene_build_host", false, tris, mat, n_tris, mats, n_mats, cam,
                     dst_host, dst_bytes, needed);
}
