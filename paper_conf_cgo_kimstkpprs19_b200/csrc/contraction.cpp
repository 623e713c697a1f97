// contraction.cpp — parser / classifier / fusion for libtc (rows a1, a2).
// Grammar: TCCG "abcd-aebf-dfce" (C-A-B, one letter per index) and the bracket
// form "C[a,b,c,d] = A[a,e,b,f] * B[d,f,c,e]".  Index property P:L64.
#include "contraction.hpp"

#include <cctype>
#include <cstring>
#include <map>

namespace tc {
namespace {

struct Lexer {
  const char *s;
  size_t i = 0;
  explicit Lexer(const char *p) : s(p) {}
  void ws() { while (s[i] && std::isspace((unsigned char)s[i])) i++; }
  char peek() { ws(); return s[i]; }
  bool eat(char c) { if (peek() == c) { i++; return true; } return false; }
  bool ident(std::string &out) {
    ws();
    size_t j = i;
    if (!(std::isalpha((unsigned char)s[j]) || s[j] == '_')) return false;
    while (std::isalnum((unsigned char)s[j]) || s[j] == '_') j++;
    out.assign(s + i, j - i);
    i = j;
    return true;
  }
  bool end() { ws(); return s[i] == 0; }
};

// Parsed lists of names per tensor.
using Lists = std::vector<std::string>[3];

bool parse_bracket(const char *e, Lists &L) {
  Lexer lx(e);
  for (int t = 0; t < 3; t++) {
    std::string tname;
    if (!lx.ident(tname) || !lx.eat('[')) return false;
    if (!lx.eat(']')) {
      for (;;) {
        std::string nm;
        if (!lx.ident(nm)) return false;
        L[t].push_back(nm);
        if (lx.eat(',')) continue;
        if (lx.eat(']')) break;
        return false;
      }
    }
    if (t == 0 && !lx.eat('=')) return false;
    if (t == 1 && !lx.eat('*')) return false;
  }
  return lx.end();
}

bool parse_tccg(const char *e, Lists &L) {
  std::string s(e);
  // trim
  size_t a = 0, b = s.size();
  while (a < b && std::isspace((unsigned char)s[a])) a++;
  while (b > a && std::isspace((unsigned char)s[b - 1])) b--;
  s = s.substr(a, b - a);
  int t = 0;
  std::string cur;
  for (char ch : s) {
    if (ch == '-') {
      if (cur.empty() || t >= 2) return false;
      for (char x : cur) L[t].push_back(std::string(1, x));
      cur.clear();
      t++;
    } else if (std::isalpha((unsigned char)ch)) {
      cur.push_back(ch);
    } else {
      return false;
    }
  }
  if (t != 2 || cur.empty()) return false;
  for (char x : cur) L[2].push_back(std::string(1, x));
  return true;
}

}  // namespace

Status parse(const char *expr, const char *extents, Contraction &out, std::string &err) {
  out = Contraction();
  if (!expr || !extents) { err = "NULL expression or extents"; return ST_INVALID_ARG; }
  Lists L;
  bool ok = std::strchr(expr, '[') ? parse_bracket(expr, L) : parse_tccg(expr, L);
  if (!ok) { err = std::string("cannot parse expression '") + expr + "'"; return ST_PARSE; }
  // limits
  std::map<std::string, int> count;
  std::vector<std::string> order;
  for (int t = 0; t < 3; t++)
    for (auto &nm : L[t]) {
      if (!count.count(nm)) order.push_back(nm);
      count[nm]++;
    }
  for (int t = 0; t < 3; t++)
    if ((int)L[t].size() > kMaxRank) { err = "tensor rank > 8"; return ST_UNSUPPORTED; }
  if ((int)order.size() > kMaxIdx) { err = "more than 16 distinct indices"; return ST_UNSUPPORTED; }
  // repeated index inside one tensor
  for (int t = 0; t < 3; t++)
    for (size_t i = 0; i < L[t].size(); i++)
      for (size_t j = i + 1; j < L[t].size(); j++)
        if (L[t][i] == L[t][j]) { err = "index '" + L[t][i] + "' repeated in one tensor"; return ST_INDEX; }
  // each index in exactly two tensors, or in all three (a batch index, R31)
  for (auto &nm : order)
    if (count[nm] != 2 && count[nm] != 3) {
      err = "index '" + nm + "' must occur in exactly two tensors, or in all three (found " +
            std::to_string(count[nm]) + ")";
      return ST_INDEX;
    }
  // extents syntax
  std::vector<std::pair<std::string, long long>> ent;
  {
    Lexer lx(extents);
    for (;;) {
      lx.ws();
      if (lx.end()) break;
      if (lx.eat(';')) continue;
      std::string nm;
      if (!lx.ident(nm) || !lx.eat(':')) { err = "malformed extents string"; return ST_PARSE; }
      lx.ws();
      bool neg = false;
      if (lx.s[lx.i] == '+' || lx.s[lx.i] == '-') { neg = lx.s[lx.i] == '-'; lx.i++; }
      if (!std::isdigit((unsigned char)lx.s[lx.i])) { err = "malformed extent value"; return ST_PARSE; }
      long long v = 0;
      bool big = false;
      while (std::isdigit((unsigned char)lx.s[lx.i])) {
        if (v > 100000000000000LL) big = true; else v = v * 10 + (lx.s[lx.i] - '0');
        lx.i++;
      }
      if (big) v = INT64_MAX;
      char nx = lx.peek();
      if (nx != ';' && nx != 0) { err = "malformed extents string"; return ST_PARSE; }
      ent.push_back({nm, neg ? -v : v});
    }
  }
  std::map<std::string, long long> ext;
  for (auto &e : ent) {
    if (!count.count(e.first)) { err = "extent for unknown index '" + e.first + "'"; return ST_INDEX; }
    if (ext.count(e.first)) { err = "extent for '" + e.first + "' given twice"; return ST_INDEX; }
    ext[e.first] = e.second;
  }
  for (auto &nm : order)
    if (!ext.count(nm)) { err = "no extent for index '" + nm + "'"; return ST_INDEX; }
  for (auto &nm : order)
    if (ext[nm] < 1) { err = "extent of '" + nm + "' must be >= 1"; return ST_EXTENT; }
  {
    // the whole iteration space (and hence every tensor) must count in int64
    unsigned __int128 all = 1;
    for (auto &nm : order) {
      all *= (unsigned __int128)ext[nm];
      if (all >= ((unsigned __int128)1 << 63)) { err = "element count overflows int64"; return ST_EXTENT; }
    }
  }
  // build
  for (auto &nm : order) {
    Index I;
    I.name = nm;
    I.n = ext[nm];
    out.ix.push_back(I);
  }
  auto id_of = [&](const std::string &nm) {
    for (size_t i = 0; i < order.size(); i++) if (order[i] == nm) return (int)i;
    return -1;
  };
  for (int t = 0; t < 3; t++) {
    int64_t st = 1;
    for (auto &nm : L[t]) {
      int id = id_of(nm);
      out.t[t].idx.push_back(id);
      out.t[t].stride.push_back(st);
      st *= out.ix[id].n;
    }
    out.parent_numel[t] = st;
  }
  for (size_t id = 0; id < out.ix.size(); id++) {
    bool inC = out.pos_in(0, (int)id) >= 0, inA = out.pos_in(1, (int)id) >= 0;
    const bool inB = out.pos_in(2, (int)id) >= 0;
    out.ix[id].cls = !inC ? INTL : (inA && inB ? BATCH : inA ? EXT_A : EXT_B);
  }
  return ST_OK;
}

static void remove_index(Contraction &c, int id) {
  for (int t = 0; t < 3; t++) {
    auto &v = c.t[t];
    for (size_t k = 0; k < v.idx.size(); k++)
      if (v.idx[k] == id) {
        v.idx.erase(v.idx.begin() + k);
        v.stride.erase(v.stride.begin() + k);
        break;
      }
    for (auto &x : v.idx) if (x > id) x--;
  }
  c.ix.erase(c.ix.begin() + id);
}

void normalize(Contraction &c, bool fuse) {
  // drop extent-1 indices (they contribute one term / one element)
  for (int id = (int)c.ix.size() - 1; id >= 0; id--)
    if (c.ix[id].n == 1) remove_index(c, id);
  if (!fuse) return;
  // merge j into i when, in every tensor holding i, j sits right after i with
  // stride_j == stride_i * N_i (then (i, j) behaves as one index of extent N_i * N_j)
  bool changed = true;
  while (changed) {
    changed = false;
    for (size_t i = 0; i < c.ix.size() && !changed; i++) {
      int tens[2], nt = 0;
      for (int t = 0; t < 3; t++) if (c.pos_in(t, (int)i) >= 0) tens[nt++] = t;
      if (nt != 2) continue;
      int p0 = c.pos_in(tens[0], (int)i);
      if (p0 + 1 >= (int)c.t[tens[0]].idx.size()) continue;
      int j = c.t[tens[0]].idx[p0 + 1];
      bool good = true;
      for (int q = 0; q < 2 && good; q++) {
        int t = tens[q], p = c.pos_in(t, (int)i);
        if (p + 1 >= (int)c.t[t].idx.size() || c.t[t].idx[p + 1] != j) good = false;
        else if (c.t[t].stride[p + 1] != c.t[t].stride[p] * c.ix[i].n) good = false;
      }
      // j must not live in the third tensor (same class as i)
      for (int t = 0; t < 3 && good; t++)
        if (t != tens[0] && t != tens[1] && c.pos_in(t, j) >= 0) good = false;
      // the merged extent stays below 2^31 (tile coordinates and TMA boxes count in int32)
      if (good && (long double)c.ix[i].n * (long double)c.ix[j].n > 2147483647.0L) good = false;
      if (!good) continue;
      c.ix[i].n *= c.ix[j].n;
      c.ix[i].name += "*" + c.ix[j].name;
      remove_index(c, j);
      changed = true;
    }
  }
}

bool split_large(Contraction &c, std::string &err) {
  const int64_t M = 2147483647LL;
  for (size_t i = 0; i < c.ix.size(); i++) {
    const int64_t n = c.ix[i].n;
    if (n <= M) continue;
    // smallest outer part d >= n / M dividing n (so the inner part n / d <= M is as long as
    // possible: it keeps the index's contiguous run); bounded search
    const int64_t lo = (n + M - 1) / M;
    int64_t d = 0;
    for (int64_t q = lo; q <= M && q < lo + (int64_t(1) << 24); q++)
      if (n % q == 0) { d = q; break; }
    if (!d) { err = "extent of '" + c.ix[i].name + "' exceeds 2^31-1 and has no factor pair below 2^31"; return false; }
    const int64_t inner = n / d;
    Index hi = c.ix[i];
    hi.n = d;
    hi.name = c.ix[i].name + "'";
    c.ix[i].n = inner;
    const int j = (int)c.ix.size();
    c.ix.push_back(hi);
    for (int t = 0; t < 3; t++) {
      const int p = c.pos_in(t, (int)i);
      if (p < 0) continue;
      auto &v = c.t[t];
      if ((int)v.idx.size() >= kMaxRank) { err = "splitting '" + hi.name + "' exceeds the rank limit"; return false; }
      v.idx.insert(v.idx.begin() + p + 1, j);
      v.stride.insert(v.stride.begin() + p + 1, v.stride[p] * inner);
    }
  }
  return true;
}

}  // namespace tc
