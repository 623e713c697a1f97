// contraction.hpp — expression parser, index classifier and index fusion of libtc
// (SURVEY 8(a) rows a1, a2).  Independent of oracle/ (own grammar code, own checks).
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace tc {

enum Status {
  ST_OK = 0, ST_INVALID_ARG = 1, ST_PARSE = 2, ST_INDEX = 3, ST_EXTENT = 4,
  ST_UNSUPPORTED = 5, ST_NO_CONFIG = 6, ST_CUDA = 7, ST_ALLOC = 8
};

// Reuse class of an index: each index is a reuse direction of the one tensor that
// does not contain it.
// BATCH (R31): an index of C, A and B — a Hadamard index, not
// summed; the kernels run one slab of C per batch value (grid y).
enum Cls { EXT_A = 0, EXT_B = 1, INTL = 2, BATCH = 3 };
inline bool is_ext(int cls) { return cls == EXT_A || cls == EXT_B; }

constexpr int kMaxRank = 8;
constexpr int kMaxIdx = 16;

struct Index {
  std::string name;   // original name, or "a*b*c" after fusion
  int64_t n = 1;      // extent
  int cls = INTL;
};

struct TensorView {
  std::vector<int> idx;         // index ids, position 0 = fastest varying
  std::vector<int64_t> stride;  // element stride per position
  int64_t base = 0;             // element offset of the origin (restricted plans)
};

struct Contraction {
  std::vector<Index> ix;
  TensorView t[3];              // 0 = C, 1 = A, 2 = B
  // numel of the dense parent tensors (for bounds / overlap checks and workspace sizes)
  int64_t parent_numel[3] = {1, 1, 1};

  int pos_in(int t, int id) const {
    for (size_t k = 0; k < this->t[t].idx.size(); k++)
      if (this->t[t].idx[k] == id) return (int)k;
    return -1;
  }
  int64_t stride_of(int t, int id) const {
    int p = pos_in(t, id);
    return p < 0 ? 0 : this->t[t].stride[p];
  }
  int64_t numel(int t) const {
    int64_t n = 1;
    for (int id : this->t[t].idx) n *= ix[id].n;
    return n;
  }
  // C's first non-batch index (the "C FVI" the tiling maps first), or -1
  int c_fvi() const {
    for (int id : this->t[0].idx)
      if (ix[id].cls != BATCH) return id;
    return -1;
  }
  // product of the batch extents (1 without batch indices)
  int64_t nbatch() const {
    int64_t n = 1;
    for (auto &i : ix) if (i.cls == BATCH) n *= i.n;
    return n;
  }
  double flops() const {
    double f = 2.0;
    for (auto &i : ix) f *= (double)i.n;
    return f;
  }
  // Largest element offset touched in tensor t, + 1 (span of the view).
  int64_t span(int t) const {
    int64_t s = this->t[t].base;
    for (size_t k = 0; k < this->t[t].idx.size(); k++)
      s += (ix[this->t[t].idx[k]].n - 1) * this->t[t].stride[k];
    return s + 1;
  }
};

// Parse + validate (rules: tests/golden/validation_rules.json; check order documented in
// DESIGN.md R23-R25).  Dense first-index-fastest strides.  `err` gets a detail message.
Status parse(const char *expr, const char *extents, Contraction &out, std::string &err);

// Row a2: drop extent-1 indices and merge runs of indices that are adjacent, in the same
// order and stride-compatible in every tensor holding them (exact; P:L164 mentions merging
// as a choice the paper did not consider).  Records the merge in the index name.
void normalize(Contraction &c, bool fuse);
// Row f1 ("splitting each dimension into multiple dimensions"): every index longer
// than 2^31-1 (tile coordinates, grid and TMA boxes count in int32) becomes two indices —
// inner n / d and outer d (the smallest factor >= n / (2^31-1)), stride_outer = stride_inner
// * (n / d) in every tensor holding it: an exact relabelling.  False (err set) when n has no
// such factor pair or a tensor would exceed the rank limit.
bool split_large(Contraction &c, std::string &err);

}  // namespace tc
