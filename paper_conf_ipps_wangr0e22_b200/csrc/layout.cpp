// layout.cpp — see layout.h.
#include "layout.h"

#include <algorithm>
#include <vector>

namespace micco {

namespace {

struct Sub {
  long long ext, s1, s2;
};

void strides(int r, const int32_t *d, long long *s) {
  long long acc = 1;
  for (int i = r - 1; i >= 0; --i) { s[i] = acc; acc *= d[i]; }
}

// merge adjacent sub-dims that are contiguous in both tensors
std::vector<Sub> merge(const std::vector<Sub> &in) {
  std::vector<Sub> out;
  for (const Sub &s : in) {
    if (!out.empty() && out.back().s1 == s.s1 * s.ext && out.back().s2 == s.s2 * s.ext) {
      out.back().ext *= s.ext;
      out.back().s1 = s.s1;
      out.back().s2 = s.s2;
    } else {
      out.push_back(s);
    }
  }
  return out;
}

}  // namespace

bool gemm_layout(int ra, const int32_t *dA, int rb, const int32_t *dB, int c, const int8_t *pa,
                 const int8_t *pb, GemmLayout &L) {
  long long sA[8], sB[8], sC[8];
  strides(ra, dA, sA);
  strides(rb, dB, sB);
  bool usedA[8] = {false}, usedB[8] = {false};
  for (int i = 0; i < c; ++i) { usedA[pa[i]] = true; usedB[pb[i]] = true; }
  int rd[8], nr = 0;
  std::vector<int> fa, fb;
  for (int i = 0; i < ra; ++i)
    if (!usedA[i]) { fa.push_back(i); rd[nr++] = dA[i]; }
  for (int i = 0; i < rb; ++i)
    if (!usedB[i]) { fb.push_back(i); rd[nr++] = dB[i]; }
  strides(nr, rd, sC);
  std::vector<Sub> m, n;
  for (size_t j = 0; j < fa.size(); ++j) m.push_back({dA[fa[j]], sA[fa[j]], sC[j]});
  for (size_t j = 0; j < fb.size(); ++j) n.push_back({dB[fb[j]], sB[fb[j]], sC[fa.size() + j]});
  m = merge(m);
  n = merge(n);
  if (m.size() > 2 || n.size() > 2) return false;
  L.Mo = 1; L.Mi = 1; L.sAmo = L.sAmi = L.sCmo = L.sCmi = 0;
  if (m.size() == 1) { L.Mi = (int)m[0].ext; L.sAmi = m[0].s1; L.sCmi = m[0].s2; }
  if (m.size() == 2) {
    L.Mo = (int)m[0].ext; L.sAmo = m[0].s1; L.sCmo = m[0].s2;
    L.Mi = (int)m[1].ext; L.sAmi = m[1].s1; L.sCmi = m[1].s2;
  }
  L.No = 1; L.Ni = 1; L.sBno = L.sBni = L.sCno = L.sCni = 0;
  if (n.size() == 1) { L.Ni = (int)n[0].ext; L.sBni = n[0].s1; L.sCni = n[0].s2; }
  if (n.size() == 2) {
    L.No = (int)n[0].ext; L.sBno = n[0].s1; L.sCno = n[0].s2;
    L.Ni = (int)n[1].ext; L.sBni = n[1].s1; L.sCni = n[1].s2;
  }
  // K: try every order of the contracted pairs; keep ≤ 2 sub-dims and, if possible, a
  // stride-1 inner dimension for each operand (coalesced tile loads).
  int perm[8];
  for (int i = 0; i < c; ++i) perm[i] = i;
  double best = 1e30;
  std::vector<Sub> bestK;
  do {
    std::vector<Sub> k;
    for (int i = 0; i < c; ++i) k.push_back({dA[pa[perm[i]]], sA[pa[perm[i]]], sB[pb[perm[i]]]});
    k = merge(k);
    if (k.size() > 2) continue;
    const Sub &in = k.back();
    bool coalA = in.s1 == 1 || L.sAmi == 1;
    bool coalB = in.s2 == 1 || L.sBni == 1;
    double score = (coalA ? 0 : 1) + (coalB ? 0 : 1) + 0.01 * (double)k.size();
    if (score < best) { best = score; bestK = k; }
  } while (std::next_permutation(perm, perm + c));
  if (bestK.empty()) return false;
  L.Ko = 1; L.sAko = L.sBko = 0;
  if (bestK.size() == 2) { L.Ko = (int)bestK[0].ext; L.sAko = bestK[0].s1; L.sBko = bestK[0].s2; }
  L.Ki = (int)bestK.back().ext; L.sAki = bestK.back().s1; L.sBki = bestK.back().s2;
  long long ea = 1, eb = 1, ec = 1;
  for (int i = 0; i < ra; ++i) ea *= dA[i];
  for (int i = 0; i < rb; ++i) eb *= dB[i];
  for (int i = 0; i < nr; ++i) ec *= rd[i];
  L.sliceA = ea; L.sliceB = eb; L.sliceC = ec;
  return true;
}

int gemm_class(const GemmLayout &L) {
  const bool a_mk = L.sAki == 1 || L.Ki == 1, a_km = L.sAmi == 1 || L.Mi == 1;
  const bool b_kn = L.sBni == 1 || L.Ni == 1, b_nk = L.sBki == 1 || L.Ki == 1;
  if (!(a_mk || a_km) || !(b_kn || b_nk)) return 4;
  return (a_mk ? 0 : 2) + (b_kn ? 0 : 1);
}

bool dot_layout(int ra, const int32_t *dA, int rb, const int32_t *dB, int c, const int8_t *pa,
                const int8_t *pb, DotLayout &L) {
  long long sA[8], sB[8];
  strides(ra, dA, sA);
  L.nO = 0;
  for (int i = 0; i < 3; ++i) { L.O[i] = 1; L.sAo[i] = 0; L.sBo[i] = 0; }
  L.Y = 1; L.sAy = L.sBy = 0;
  long long ea = 1;
  for (int i = 0; i < ra; ++i) ea *= dA[i];
  L.sliceA = ea;
  if (rb == 0) {  // meson trace
    if (ra != 2 || dA[0] != dA[1]) return false;
    L.mode = 2;
    L.X = dA[0];
    L.sAx = sA[0] + sA[1];
    L.sBx = 0;
    L.sliceB = 0;
    return true;
  }
  if (ra != rb || c != ra) return false;
  strides(rb, dB, sB);
  L.sliceB = ea;
  int posb[8];  // B position paired with A leg i
  for (int i = 0; i < c; ++i) posb[pa[i]] = pb[i];
  if (posb[ra - 1] == rb - 1) {
    std::vector<Sub> legs;
    for (int i = 0; i < ra; ++i) legs.push_back({dA[i], sA[i], sB[posb[i]]});
    legs = merge(legs);
    if (legs.size() > 4) return false;
    L.mode = 0;
    L.X = (int)legs.back().ext;
    L.sAx = legs.back().s1;
    L.sBx = legs.back().s2;
    int no = (int)legs.size() - 1;
    // outer legs right-aligned into O[0..2] (O[2] fastest)
    for (int j = 0; j < no; ++j) {
      int slot = 3 - no + j;
      L.O[slot] = (int)legs[j].ext; L.sAo[slot] = legs[j].s1; L.sBo[slot] = legs[j].s2;
    }
    L.nO = no;
    return true;
  }
  int jy = -1;
  for (int i = 0; i < ra; ++i)
    if (posb[i] == rb - 1) jy = i;
  L.mode = 1;
  L.X = dA[ra - 1];
  L.sAx = sA[ra - 1];
  L.sBx = sB[posb[ra - 1]];
  L.Y = dA[jy];
  L.sAy = sA[jy];
  L.sBy = sB[posb[jy]];
  int no = 0;
  for (int i = 0; i < ra; ++i) {
    if (i == ra - 1 || i == jy) continue;
    if (no >= 3) return false;
    L.O[no] = dA[i]; L.sAo[no] = sA[i]; L.sBo[no] = sB[posb[i]];
    ++no;
  }
  // kernel decomposes o as (o0, o1, o2) with O[2] fastest: right-align
  if (no < 3) {
    for (int j = no - 1; j >= 0; --j) {
      int slot = 3 - no + j;
      L.O[slot] = L.O[j]; L.sAo[slot] = L.sAo[j]; L.sBo[slot] = L.sBo[j];
    }
    for (int j = 0; j < 3 - no; ++j) { L.O[j] = 1; L.sAo[j] = 0; L.sBo[j] = 0; }
  }
  L.nO = no;
  return true;
}

}  // namespace micco
