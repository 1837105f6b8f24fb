// host_setup.cpp -- step a-0 (see host_setup.h).  Host-only C++17; no CUDA.
#include "host_setup.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <climits>
#include <cstdlib>
#include <cstring>
#include <new>
#include <functional>
#include <map>
#include <unordered_map>
#include <unordered_set>

namespace landau {
namespace {

// ---------------------------------------------------------------------------------------------
// 1D building blocks
// ---------------------------------------------------------------------------------------------
void gauss_legendre(int n, std::vector<double> &x, std::vector<double> &w) {
  x.assign(n, 0.0);
  w.assign(n, 0.0);
  const double pi = 3.14159265358979323846;
  for (int i = 0; i < (n + 1) / 2; i++) {
    double t = std::cos(pi * (i + 0.75) / (n + 0.5)), dp = 1.0;
    for (int it = 0; it < 100; it++) {
      double p0 = 1.0, p1 = t;
      for (int k = 2; k <= n; k++) {
        double p2 = ((2.0 * k - 1.0) * t * p1 - (k - 1.0) * p0) / k;
        p0 = p1;
        p1 = p2;
      }
      if (n == 1) p0 = 1.0, p1 = t;
      dp = n * (t * p1 - p0) / (t * t - 1.0);
      double dt = p1 / dp;
      t -= dt;
      if (std::fabs(dt) < 1e-17) break;
    }
    double p0 = 1.0, p1 = t;
    for (int k = 2; k <= n; k++) {
      double p2 = ((2.0 * k - 1.0) * t * p1 - (k - 1.0) * p0) / k;
      p0 = p1;
      p1 = p2;
    }
    dp = n * (t * p1 - p0) / (t * t - 1.0);
    double wt = 2.0 / ((1.0 - t * t) * dp * dp);
    x[i] = -t;
    x[n - 1 - i] = t;
    w[i] = w[n - 1 - i] = wt;
  }
  if (n % 2 == 1) x[n / 2] = 0.0;
}

// equispaced Lagrange basis on [-1, 1] (nodes -1 + 2k/p): value and derivative
double lagrange(int p, int a, double x) {
  double v = 1.0;
  for (int k = 0; k <= p; k++)
    if (k != a) v *= (x - (-1.0 + 2.0 * k / p)) / (2.0 * (a - k) / p);
  return v;
}
double lagrange_d(int p, int a, double x) {
  double s = 0.0;
  for (int m = 0; m <= p; m++) {
    if (m == a) continue;
    double v = 1.0 / (2.0 * (a - m) / p);
    for (int k = 0; k <= p; k++)
      if (k != a && k != m) v *= (x - (-1.0 + 2.0 * k / p)) / (2.0 * (a - k) / p);
    s += v;
  }
  return s;
}

inline uint64_t key2(int64_t ir, int64_t iz) { return (uint64_t(iz) << 32) | uint64_t(ir); }

struct ICell {
  int64_t R0, Z0, H;   // in units of the grid's smallest cell size; Z0 measured from z = -R
  int level;           // H = 2^(L - level)
};

}  // namespace

std::string build_plan(int ngrids, const int64_t *ncells, const double *cells, const double *radius, int order,
                       Plan &plan) {
  char msg[256];
  // fault injection for the CPU test of the C ABI's exception safety (tests/test_abi.py): a host
  // allocation failure inside the plan must come back as LANDAU_ENOMEM, not terminate the caller
  if (const char *e = getenv("LANDAU_TEST_FAIL_ALLOC"))
    if (!strcmp(e, "plan")) throw std::bad_alloc();
  const int p = order, nq = order + 1, nb = (p + 1) * (p + 1), nqp = nq * nq;
  plan = Plan();
  plan.p = p;
  plan.nq = nq;
  plan.nb = nb;
  plan.nqp = nqp;
  plan.ngrids = ngrids;
  // reference tables
  std::vector<double> xg, wg;
  gauss_legendre(nq, xg, wg);
  plan.tab_phi.resize(nqp * nb);
  plan.tab_dxi.resize(nqp * nb);
  plan.tab_deta.resize(nqp * nb);
  plan.tab1_L.resize(nq * (p + 1));   // 1-D factors [Gauss point i][node a] (element_sf_kernel)
  plan.tab1_D.resize(nq * (p + 1));
  for (int i = 0; i < nq; i++)
    for (int a = 0; a <= p; a++) {
      plan.tab1_L[i * (p + 1) + a] = lagrange(p, a, xg[i]);
      plan.tab1_D[i * (p + 1) + a] = lagrange_d(p, a, xg[i]);
    }
  for (int qz = 0; qz < nq; qz++)
    for (int qr = 0; qr < nq; qr++)
      for (int b = 0; b <= p; b++)
        for (int a = 0; a <= p; a++) {
          int q = qz * nq + qr, n = b * (p + 1) + a;
          plan.tab_phi[q * nb + n] = lagrange(p, a, xg[qr]) * lagrange(p, b, xg[qz]);
          plan.tab_dxi[q * nb + n] = lagrange_d(p, a, xg[qr]) * lagrange(p, b, xg[qz]);
          plan.tab_deta[q * nb + n] = lagrange(p, a, xg[qr]) * lagrange_d(p, b, xg[qz]);
        }

  int64_t c0 = 0, pt0 = 0;
  plan.grids.resize(ngrids);
  for (int g = 0; g < ngrids; g++) {
    GridPlan &G = plan.grids[g];
    const double R = radius[g];
    const int64_t n = ncells[g];
    if (!(R > 0) || n < 2) {
      snprintf(msg, sizeof msg, "grid %d: radius must be > 0 and the grid needs >= 2 cells", g);
      return msg;
    }
    G.R = R;
    G.cell0 = c0;
    G.ncell = n;
    G.pt0 = pt0;
    const double *cc = cells + 3 * c0;
    // ---- integer quadtree coordinates -------------------------------------------------------
    double hmin = 1e300;
    for (int64_t c = 0; c < n; c++) {
      if (!(cc[3 * c + 2] > 0) || cc[3 * c] < 0) {
        snprintf(msg, sizeof msg, "grid %d cell %lld: h must be > 0 and r0 >= 0", g, (long long)c);
        return msg;
      }
      hmin = std::min(hmin, cc[3 * c + 2]);
    }
    const double rootH = R / hmin;
    const int L = (int)std::llround(std::log2(rootH));
    if (L < 0 || L > 26 || std::fabs(std::ldexp(1.0, L) - rootH) > 1e-9 * rootH) {
      snprintf(msg, sizeof msg, "grid %d: cell sizes are not R / 2^k", g);
      return msg;
    }
    std::vector<ICell> ic(n);
    std::unordered_set<uint64_t> present;   // (level, R0/H, Z0/H)
    auto qkey = [](int level, int64_t i, int64_t j) { return (uint64_t(level) << 58) | (uint64_t(j) << 29) | uint64_t(i); };
    int64_t area = 0;
    const int64_t Rl = int64_t(1) << L;
    for (int64_t c = 0; c < n; c++) {
      double a = cc[3 * c] / hmin, b = (cc[3 * c + 1] + R) / hmin, h = cc[3 * c + 2] / hmin;
      ICell &x = ic[c];
      x.R0 = std::llround(a);
      x.Z0 = std::llround(b);
      x.H = std::llround(h);
      int lv = L - (int)std::llround(std::log2((double)x.H));
      x.level = lv;
      bool ok = std::fabs(a - x.R0) < 1e-6 && std::fabs(b - x.Z0) < 1e-6 && std::fabs(h - x.H) < 1e-6 && x.H >= 1 &&
                (x.H & (x.H - 1)) == 0 && lv >= 0 && x.R0 % x.H == 0 && x.Z0 % x.H == 0 && x.R0 + x.H <= Rl &&
                x.Z0 + x.H <= 2 * Rl && x.Z0 >= 0;
      if (!ok) {
        snprintf(msg, sizeof msg, "grid %d cell %lld is not a quadtree cell of [0,R]x[-R,R]", g, (long long)c);
        return msg;
      }
      if (!present.insert(qkey(lv, x.R0 / x.H, x.Z0 / x.H)).second) {
        snprintf(msg, sizeof msg, "grid %d: duplicate cell %lld", g, (long long)c);
        return msg;
      }
      area += x.H * x.H;
    }
    for (int64_t c = 0; c < n; c++) {   // no ancestor of a leaf may itself be a leaf
      const ICell &x = ic[c];
      for (int lv = x.level - 1; lv >= 0; lv--) {
        int64_t H = int64_t(1) << (L - lv);
        if (present.count(qkey(lv, x.R0 / H, x.Z0 / H))) {
          snprintf(msg, sizeof msg, "grid %d: overlapping cells", g);
          return msg;
        }
      }
    }
    if (area != 2 * Rl * Rl) {
      snprintf(msg, sizeof msg, "grid %d: cells do not tile [0,R]x[-R,R]", g);
      return msg;
    }
    // 2:1 edge balance: the leaf across each edge of a cell is at most twice its size
    auto leaf_size = [&](int64_t x2, int64_t z2) -> int64_t {   // doubled coords of an interior point
      if (x2 < 0 || z2 < 0 || x2 >= 2 * Rl || z2 >= 4 * Rl) return 0;
      for (int lv = L; lv >= 0; lv--) {
        int64_t H = int64_t(1) << (L - lv);
        if (present.count(qkey(lv, (x2 / 2) / H, (z2 / 2) / H))) return H;
      }
      return -1;
    };
    for (int64_t c = 0; c < n; c++) {
      const ICell &x = ic[c];
      int64_t pts[4][2] = {{2 * (x.R0 + x.H) + 1, 2 * x.Z0 + 1}, {2 * x.R0 - 1, 2 * x.Z0 + 1},
                           {2 * x.R0 + 1, 2 * (x.Z0 + x.H) + 1}, {2 * x.R0 + 1, 2 * x.Z0 - 1}};
      for (auto &q : pts) {
        int64_t s = leaf_size(q[0], q[1]);
        if (s > 2 * x.H) {
          snprintf(msg, sizeof msg, "grid %d: quadtree not 2:1 balanced at cell %lld", g, (long long)c);
          return msg;
        }
      }
    }
    // ---- node positions (lattice unit hmin / p) ------------------------------------------------
    std::unordered_map<uint64_t, int> pos_id;   // candidate positions
    std::vector<std::pair<int64_t, int64_t>> pos;   // (ir, iz)
    pos_id.reserve(n * nb);
    std::vector<int> cell_node(n * nb);
    for (int64_t c = 0; c < n; c++)
      for (int b = 0; b <= p; b++)
        for (int a = 0; a <= p; a++) {
          int64_t ir = ic[c].R0 * p + a * ic[c].H, iz = ic[c].Z0 * p + b * ic[c].H;
          auto it = pos_id.emplace(key2(ir, iz), (int)pos.size());
          if (it.second) pos.emplace_back(ir, iz);
          cell_node[c * nb + b * (p + 1) + a] = it.first->second;
        }
    // hanging positions: odd multiples of H/2 on a cell edge that some finer neighbour has as node
    struct Hang {
      int64_t mr[8], mz[8];
      double mw[8];
    };
    std::unordered_map<int, Hang> hang;
    for (int64_t c = 0; c < n; c++) {
      const ICell &x = ic[c];
      if (x.H < 2) continue;
      const int64_t h2 = x.H / 2, r0 = x.R0 * p, z0 = x.Z0 * p, Lp = x.H * p;
      // edges: (start point, direction)
      const int64_t E[4][4] = {{r0, z0, 1, 0}, {r0, z0 + Lp, 1, 0}, {r0, z0, 0, 1}, {r0 + Lp, z0, 0, 1}};
      for (auto &e : E) {
        for (int k = 1; k < 2 * p; k += 2) {
          int64_t ir = e[0] + e[2] * k * h2, iz = e[1] + e[3] * k * h2;
          auto it = pos_id.find(key2(ir, iz));
          if (it == pos_id.end()) continue;
          Hang hg;
          for (int j = 0; j <= p; j++) {
            hg.mr[j] = e[0] + e[2] * j * x.H;
            hg.mz[j] = e[1] + e[3] * j * x.H;
            // L_j(t), t = k / (2p), nodes i/p: prod_{i != j} (k - 2i) / (2 (j - i)) -- exact integers
            double num = 1.0, den = 1.0;
            for (int i = 0; i <= p; i++)
              if (i != j) num *= double(k - 2 * i), den *= double(2 * (j - i));
            hg.mw[j] = num / den;
          }
          hang[it->second] = hg;
        }
      }
    }
    // DOFs: non-hanging positions sorted by (iz, ir)
    std::vector<int> order_;
    for (int i = 0; i < (int)pos.size(); i++)
      if (!hang.count(i)) order_.push_back(i);
    std::sort(order_.begin(), order_.end(), [&](int a, int b) {
      return pos[a].second != pos[b].second ? pos[a].second < pos[b].second : pos[a].first < pos[b].first;
    });
    std::vector<int> dof_of(pos.size(), -1);
    G.ndof = (int)order_.size();
    G.node_r.resize(G.ndof);
    G.node_z.resize(G.ndof);
    const double unit = hmin / p;
    for (int d = 0; d < G.ndof; d++) {
      dof_of[order_[d]] = d;
      G.node_r[d] = pos[order_[d]].first * unit;
      G.node_z[d] = pos[order_[d]].second * unit - R;
    }
    // resolve a position into (dof, weight) terms (recursive through constraints)
    std::function<void(int, double, std::vector<std::pair<int, double>> &, int)> resolve =
        [&](int pid, double s, std::vector<std::pair<int, double>> &out, int depth) {
          if (dof_of[pid] >= 0) {
            for (auto &t : out)
              if (t.first == dof_of[pid]) {
                t.second += s;
                return;
              }
            out.emplace_back(dof_of[pid], s);
            return;
          }
          if (depth > 8) return;
          const Hang &hg = hang.at(pid);
          for (int j = 0; j <= p; j++) {
            if (hg.mw[j] == 0.0) continue;
            auto it = pos_id.find(key2(hg.mr[j], hg.mz[j]));
            if (it == pos_id.end()) continue;   // cannot happen for a tiled, balanced tree
            resolve(it->second, s * hg.mw[j], out, depth + 1);
          }
        };
    // ---- per-cell extraction ----------------------------------------------------------------
    G.ne.resize(n);
    G.edof_off.assign(n + 1, 0);
    G.P_off.assign(n + 1, 0);
    std::vector<std::vector<std::pair<int, double>>> loc(nb);
    for (int64_t c = 0; c < n; c++) {
      std::vector<int> d;
      for (int a = 0; a < nb; a++) {
        loc[a].clear();
        resolve(cell_node[c * nb + a], 1.0, loc[a], 0);
        if (loc[a].empty()) {
          snprintf(msg, sizeof msg, "grid %d: unresolvable node in cell %lld", g, (long long)c);
          return msg;
        }
        for (auto &t : loc[a]) d.push_back(t.first);
        // field extraction list (global over grids)
        plan.ext_ptr.push_back((int32_t)plan.ext_dof.size());
        for (auto &t : loc[a]) {
          plan.ext_dof.push_back(t.first);
          plan.ext_w.push_back(t.second);
        }
      }
      std::sort(d.begin(), d.end());
      d.erase(std::unique(d.begin(), d.end()), d.end());
      int ne = (int)d.size();
      G.ne[c] = ne;
      G.edof_off[c + 1] = G.edof_off[c] + ne;
      G.edof.insert(G.edof.end(), d.begin(), d.end());
      G.P_off[c + 1] = G.P_off[c] + (int64_t)nb * ne;
      size_t base = G.P.size();
      G.P.resize(base + (size_t)nb * ne, 0.0);
      for (int a = 0; a < nb; a++)
        for (auto &t : loc[a]) {
          int j = int(std::lower_bound(d.begin(), d.end(), t.first) - d.begin());
          G.P[base + (size_t)a * ne + j] += t.second;
        }
      G.ncoo += (int64_t)ne * ne;
    }
    // ---- CSR pattern ------------------------------------------------------------------------
    std::vector<std::vector<int>> rows(G.ndof);
    for (int64_t c = 0; c < n; c++) {
      const int *d = &G.edof[G.edof_off[c]];
      for (int i = 0; i < G.ne[c]; i++)
        for (int j = 0; j < G.ne[c]; j++) rows[d[i]].push_back(d[j]);
    }
    G.rowptr.assign(G.ndof + 1, 0);
    for (int i = 0; i < G.ndof; i++) {
      auto &r = rows[i];
      std::sort(r.begin(), r.end());
      r.erase(std::unique(r.begin(), r.end()), r.end());
      G.rowptr[i + 1] = G.rowptr[i] + (int64_t)r.size();
      G.col.insert(G.col.end(), r.begin(), r.end());
    }
    // ---- RCM ordering and band map (NEXT-2) ---------------------------------------------------
    // reverse Cuthill-McKee: BFS from a pseudo-peripheral node, neighbours by increasing degree,
    // every connected component in turn, then the order reversed (PAPER.md:1@25294, [23])
    {
      const int n = G.ndof;
      std::vector<int> deg(n);
      for (int i = 0; i < n; i++) deg[i] = (int)(G.rowptr[i + 1] - G.rowptr[i]);
      auto bfs = [&](int root, std::vector<int> &order, std::vector<int> &level, std::vector<char> &seen) {
        order.clear();
        order.push_back(root);
        seen[root] = 1;
        level[root] = 0;
        for (size_t h = 0; h < order.size(); h++) {
          const int u = order[h];
          std::vector<int> nb;
          for (int64_t q = G.rowptr[u]; q < G.rowptr[u + 1]; q++) {
            const int v = G.col[q];
            if (!seen[v]) nb.push_back(v);
          }
          std::sort(nb.begin(), nb.end(), [&](int a, int b) { return deg[a] != deg[b] ? deg[a] < deg[b] : a < b; });
          for (int v : nb)
            if (!seen[v]) {
              seen[v] = 1;
              level[v] = level[u] + 1;
              order.push_back(v);
            }
        }
      };
      std::vector<char> done(n, 0);
      std::vector<int> cm, level(n, 0), order;
      for (int start = 0; start < n; start++) {
        if (done[start]) continue;
        // pseudo-peripheral root (George-Liu): repeat BFS from a min-degree node of the last level
        int root = start;
        int last_depth = -1;
        for (int it = 0; it < 8; it++) {
          std::vector<char> seen(done);
          bfs(root, order, level, seen);
          const int depth = level[order.back()];
          if (depth <= last_depth) break;
          last_depth = depth;
          int best = order.back();
          for (int v : order)
            if (level[v] == depth && deg[v] < deg[best]) best = v;
          root = best;
        }
        std::vector<char> seen(done);
        bfs(root, order, level, seen);
        for (int v : order) {
          done[v] = 1;
          cm.push_back(v);
        }
      }
      // connected grids up to 2048 DOFs: the Cuthill-McKee order from EVERY root, keep the smallest
      // bandwidth (George-Liu's pseudo-peripheral root is a heuristic: 81 on the C2/C4 grid against
      // 78 for the best root, and the band kernel's window is B + 2 rounded up to 8: 88 -> 80, 17%
      // fewer FLOP per step).  A root is abandoned as soon as its partial order reaches the best B.
      if ((int)cm.size() == n && n > 1 && n <= 2048 && !getenv("LANDAU_RCM_PERIPHERAL")) {
        std::vector<int> sadj(G.col.size());   // neighbours by (degree, id), self excluded below
        for (int i = 0; i < n; i++) {
          std::copy(G.col.begin() + G.rowptr[i], G.col.begin() + G.rowptr[i + 1], sadj.begin() + G.rowptr[i]);
          std::sort(sadj.begin() + G.rowptr[i], sadj.begin() + G.rowptr[i + 1],
                    [&](int a, int b) { return deg[a] != deg[b] ? deg[a] < deg[b] : a < b; });
        }
        auto band_of = [&](const std::vector<int> &ord, std::vector<int> &pos) {
          for (int k = 0; k < n; k++) pos[ord[k]] = k;
          int b = 0;
          for (int i = 0; i < n; i++)
            for (int64_t q = G.rowptr[i]; q < G.rowptr[i + 1]; q++) b = std::max(b, std::abs(pos[i] - pos[G.col[q]]));
          return b;
        };
        std::vector<int> pos(n, -1), ord, best = cm;
        int bestB = band_of(cm, pos);
        ord.reserve(n);
        for (int root = 0; root < n; root++) {
          std::fill(pos.begin(), pos.end(), -1);
          ord.clear();
          ord.push_back(root);
          pos[root] = 0;
          bool cut = false;
          for (size_t h = 0; h < ord.size() && !cut; h++) {
            const int u = ord[h];
            for (int64_t q = G.rowptr[u]; q < G.rowptr[u + 1]; q++) {
              const int v = sadj[q];
              if (pos[v] >= 0) continue;
              pos[v] = (int)ord.size();
              ord.push_back(v);
              // u is v's lowest-placed neighbour (BFS), so this edge is v's widest to the front
              if (pos[v] - (int)h >= bestB) {
                cut = true;
                break;
              }
            }
          }
          if (cut || (int)ord.size() != n) continue;
          bestB = band_of(ord, pos);
          best = ord;
        }
        cm = best;
      }
      G.rcm_perm.assign(cm.rbegin(), cm.rend());
      G.rcm_iperm.assign(n, 0);
      for (int k = 0; k < n; k++) G.rcm_iperm[G.rcm_perm[k]] = k;
      int B = 0, B0 = 0;
      for (int i = 0; i < n; i++)
        for (int64_t q = G.rowptr[i]; q < G.rowptr[i + 1]; q++) {
          B = std::max(B, std::abs(G.rcm_iperm[i] - G.rcm_iperm[G.col[q]]));
          B0 = std::max(B0, std::abs(i - G.col[q]));
        }
      if (B0 < B) {   // tiny meshes: the (z, r) numbering can beat RCM; keep the smaller band
        for (int k = 0; k < n; k++) G.rcm_perm[k] = G.rcm_iperm[k] = k;
        B = B0;
      }
      G.band = B;
      // entering-row entry lists (see host_setup.h); the pattern is symmetric, so A(j, i) is the CSR
      // entry (perm j, perm i), found by a binary search in its sorted row
      auto slot_of = [&](int r, int c) -> int32_t {
        const int *b = G.col.data() + G.rowptr[r], *e = G.col.data() + G.rowptr[r + 1];
        const int *f = std::lower_bound(b, e, c);
        return (f != e && *f == c) ? (int32_t)(f - G.col.data()) : -1;
      };
      // the factorisation runs a window of P = Bp + 1 rows, P a multiple of 8 (kernels_band.cuh):
      // positions are relative to the padded half-bandwidth Bp >= B (entries past B are zero)
      const int Bp = (B + 2 + 7) / 8 * 8 - 1;   // B + 2 <= P: the rank-2 kernel's row k+1 fits the window
      G.band_p = Bp;
      G.ent_ptr.assign(1, 0);
      G.ent_slot.clear();
      G.ent_pos.clear();
      G.ent_max = 0;
      std::vector<std::pair<int, int32_t>> ent;
      for (int ni = 0; ni < n; ni++) {
        const int oi = G.rcm_perm[ni];
        ent.clear();
        for (int64_t q = G.rowptr[oi]; q < G.rowptr[oi + 1]; q++) {
          const int nj = G.rcm_iperm[G.col[q]];
          if (nj <= ni) ent.push_back({nj - ni + Bp, (int32_t)q});                         // A(i, j), row part
          if (nj < ni) ent.push_back({Bp + 1 + nj - ni + Bp, slot_of(G.col[q], oi)});      // A(j, i), column part
        }
        std::sort(ent.begin(), ent.end());
        for (auto &e : ent) {
          if (e.second < 0) return "band: CSR pattern is not symmetric";
          // kernel layout (band_lu2_kernel): row-in-group * 4P, row part p in [0, P), column part
          // at 2P + (p - P) (each stored twice by the kernel, the copy at +P)
          const int P = Bp + 1, p = e.first;
          G.ent_pos.push_back((uint16_t)((ni % 8) * 4 * P + (p < P ? p : 2 * P + p - P)));
          G.ent_slot.push_back(e.second);
        }
        G.ent_max = std::max(G.ent_max, (int)ent.size());
        G.ent_ptr.push_back((int32_t)G.ent_slot.size());
      }
    }
    // ---- gather maps --------------------------------------------------------------------------
    // slot contributions: (cell, a, b) with P[a][i] P[b][j] != 0, in (cell, a, b) order
    GatherMap csr, coo;
    std::vector<std::vector<std::pair<int32_t, double>>> csr_slots(G.col.size());
    coo.ptr.push_back(0);
    for (int64_t c = 0; c < n; c++) {
      const int ne = G.ne[c];
      const int *d = &G.edof[G.edof_off[c]];
      const double *Pc = &G.P[G.P_off[c]];
      const int64_t ge = c0 + c;
      std::vector<int64_t> slot(ne * ne);
      for (int i = 0; i < ne; i++)
        for (int j = 0; j < ne; j++) {
          auto b = G.col.begin() + G.rowptr[d[i]], e = G.col.begin() + G.rowptr[d[i] + 1];
          slot[i * ne + j] = std::lower_bound(b, e, d[j]) - G.col.begin();
        }
      std::vector<std::vector<std::pair<int32_t, double>>> cslot(ne * ne);
      for (int a = 0; a < nb; a++)
        for (int bb = 0; bb < nb; bb++) {
          const int32_t idx = (int32_t)(ge * 2 * nb * nb + 2 * (a * nb + bb));   // [cell][k][l][D|K] interleaved
          for (int i = 0; i < ne; i++) {
            double pa = Pc[a * ne + i];
            if (pa == 0.0) continue;
            for (int j = 0; j < ne; j++) {
              double pb = Pc[bb * ne + j];
              if (pb == 0.0) continue;
              csr_slots[slot[i * ne + j]].emplace_back(idx, pa * pb);
              cslot[i * ne + j].emplace_back(idx, pa * pb);
            }
          }
        }
      for (auto &s : cslot) {
        for (auto &t : s) {
          coo.idx.push_back(t.first);
          coo.w.push_back(t.second);
        }
        coo.ptr.push_back((int64_t)coo.idx.size());
      }
    }
    csr.ptr.push_back(0);
    for (auto &s : csr_slots) {
      for (auto &t : s) {
        csr.idx.push_back(t.first);
        csr.w.push_back(t.second);
      }
      csr.ptr.push_back((int64_t)csr.idx.size());
    }
    plan.csr_map.push_back(std::move(csr));
    plan.coo_map.push_back(std::move(coo));
    // ---- points and per-cell data ---------------------------------------------------------------
    for (int64_t c = 0; c < n; c++) {
      const double r0 = cc[3 * c], z0 = cc[3 * c + 1], h = cc[3 * c + 2];
      plan.cell_h.push_back(h);
      plan.cell_grid.push_back(g);
      // points from the cell centre: with the exactly antisymmetric Gauss nodes (xg[n-1-i] = -xg[i])
      // the points of a mirrored cell (z0' = -z0 - h exactly, as the dyadic meshes of inputs.py give)
      // are the bit-exact negatives z' = -z, which the mirror kernels require (landau_create)
      const double rc = r0 + 0.5 * h, zc = z0 + 0.5 * h, hh = 0.5 * h;
      for (int qz = 0; qz < nq; qz++)
        for (int qr = 0; qr < nq; qr++) {
          double r = rc + hh * xg[qr];
          double z = zc + hh * xg[qz];
          plan.pr.push_back(r);
          plan.pz.push_back(z);
          plan.pw.push_back(wg[qr] * wg[qz] * (0.25 * h * h) * r);
        }
    }
    c0 += n;
    pt0 += n * nqp;
  }
  plan.ext_ptr.push_back((int32_t)plan.ext_dof.size());
  plan.ncell = c0;
  plan.npts = pt0;
  if (plan.ncell * 2 * nb * nb > INT32_MAX) return "mesh too large for 32-bit gather indices";
  return "";
}

std::string build_phase_maps(const Plan &plan, const std::vector<GatherMap> &maps, int cap, PhaseMaps &out) {
  out = PhaseMaps();
  const int nb = plan.nb;
  const int64_t csz = 2LL * nb * nb;   // doubles per cell in the element buffer
  out.grid_phase_ptr.push_back(0);
  out.slot_ptr.push_back(0);
  for (int g = 0; g < plan.ngrids; g++) {
    const GridPlan &G = plan.grids[g];
    const int nph = (int)((G.ncell + cap - 1) / cap), per = (int)((G.ncell + nph - 1) / nph);   // balanced
    const int ph0 = (int)out.cell_ptr.size();
    for (int64_t c = 0; c < G.ncell; c += per) out.cell_ptr.push_back((int32_t)(G.cell0 + c));
    out.max_cells = std::max(out.max_cells, per);
    const int ph1 = (int)out.cell_ptr.size();
    out.grid_phase_ptr.push_back(ph1);
    auto phase_of = [&](int64_t ge) { return ph0 + (int)((ge - G.cell0) / per); };
    const GatherMap &m = maps[g];
    const int64_t nslots = (int64_t)m.ptr.size() - 1;
    std::vector<int32_t> pfirst(nslots, INT32_MAX), plast(nslots, -1), xid(nslots, 0);
    int nx = 0;
    for (int64_t s = 0; s < nslots; s++) {
      for (int64_t k = m.ptr[s]; k < m.ptr[s + 1]; k++) {
        const int ph = phase_of(m.idx[k] / csz);
        if (ph < plast[s]) return "phase maps: contributions not in cell order";
        pfirst[s] = std::min(pfirst[s], ph);
        plast[s] = std::max(plast[s], ph);
      }
      if (plast[s] > pfirst[s]) xid[s] = nx++;
    }
    out.max_cross = std::max(out.max_cross, nx);
    for (int ph = ph0; ph < ph1; ph++) {
      const int64_t cbase = (int64_t)out.cell_ptr[ph];
      for (int64_t s = 0; s < nslots; s++) {
        if (ph < pfirst[s] || ph > plast[s]) continue;
        int n = 0;
        int32_t ii[4] = {0, 0, 0, 0};
        double ww[4] = {0.0, 0.0, 0.0, 0.0};
        const int32_t o0 = (int32_t)out.oidx.size();
        for (int64_t k = m.ptr[s]; k < m.ptr[s + 1]; k++) {
          const int64_t ge = m.idx[k] / csz;
          if (phase_of(ge) != ph) continue;
          const int32_t li = (int32_t)((ge - cbase) * csz + m.idx[k] % csz);
          if (n < 4) {
            ii[n] = li;
            ww[n] = m.w[k];
          } else {
            out.oidx.push_back(li);
            out.ow.push_back(m.w[k]);
          }
          n++;
        }
        const int mode = pfirst[s] == plast[s] ? 0 : ph == pfirst[s] ? 1 : ph == plast[s] ? 3 : 2;
        out.meta.push_back((int32_t)s);
        out.meta.push_back(mode | (std::min(n, 4) << 2) | (xid[s] << 5));
        for (int t = 0; t < 4; t++) {
          out.idx4.push_back(ii[t]);
          out.w4.push_back(ww[t]);
        }
        out.optr.push_back(o0);
        out.optr.push_back((int32_t)out.oidx.size());
        if (out.oidx.size() > (size_t)INT32_MAX / 2 || out.meta.size() > (size_t)INT32_MAX / 2)
          return "phase maps: too many entries";
      }
      out.slot_ptr.push_back((int32_t)(out.meta.size() / 2));
    }
  }
  out.cell_ptr.push_back((int32_t)plan.ncell);   // end of the last phase
  return "";
}

std::string build_plan3d(int ncell, int order, double R, Plan3D &P) {
  if (ncell < 1 || order < 2 || order > 3 || !(R > 0.0)) return "3d: ncell >= 1, order 2 or 3, R > 0";
  const int p = order, S = p + 1, nb = S * S * S;
  const int64_t M = (int64_t)ncell * p + 1, nc3 = (int64_t)ncell * ncell * ncell;
  if (M * M * M > INT32_MAX || nc3 * nb * nb * 2 > INT32_MAX) return "3d: grid too large";
  P = Plan3D{};
  P.ncell = ncell;
  P.p = p;
  P.s1 = S;
  P.nb = nb;
  P.R = R;
  P.h = 2.0 * R / ncell;
  P.ndof = M * M * M;
  P.npts = nc3 * nb;
  std::vector<double> xg, wg;
  gauss_legendre(S, xg, wg);
  P.L1.resize(S * S);
  P.D1.resize(S * S);
  for (int i = 0; i < S; i++)
    for (int a = 0; a < S; a++) {
      P.L1[i * S + a] = lagrange(p, a, xg[i]);
      P.D1[i * S + a] = lagrange_d(p, a, xg[i]);
    }
  P.xyz.resize(3 * P.npts);
  P.w.resize(P.npts);
  P.dofs.resize(nc3 * nb);
  const double hh = 0.5 * P.h;
  for (int64_t cz = 0; cz < ncell; cz++)
    for (int64_t cy = 0; cy < ncell; cy++)
      for (int64_t cx = 0; cx < ncell; cx++) {
        const int64_t e = (cz * ncell + cy) * ncell + cx;
        for (int k = 0; k < S; k++)
          for (int j = 0; j < S; j++)
            for (int i = 0; i < S; i++)
              P.dofs[e * nb + (k * S + j) * S + i] = (int32_t)(((cz * p + k) * M + (cy * p + j)) * M + (cx * p + i));
        for (int a = 0; a < S; a++)
          for (int b = 0; b < S; b++)
            for (int c = 0; c < S; c++) {
              const int64_t pt = e * nb + (a * S + b) * S + c;
              P.xyz[pt] = -R + P.h * cx + hh * (xg[c] + 1.0);
              P.xyz[P.npts + pt] = -R + P.h * cy + hh * (xg[b] + 1.0);
              P.xyz[2 * P.npts + pt] = -R + P.h * cz + hh * (xg[a] + 1.0);
              P.w[pt] = wg[a] * wg[b] * wg[c] * hh * hh * hh;
            }
      }
  // 1-D neighbour ranges: the lattice indices sharing a cube with i
  std::vector<int64_t> lo(M), hi(M);
  for (int64_t i = 0; i < M; i++) {
    int64_t c0 = i / p, c1 = c0;
    if (i % p == 0 && c0 > 0) c0--;
    c1 = std::min<int64_t>(c1, ncell - 1);
    lo[i] = c0 * p;
    hi[i] = (c1 + 1) * p;
  }
  P.rowptr.assign(P.ndof + 1, 0);
  for (int64_t iz = 0; iz < M; iz++)
    for (int64_t iy = 0; iy < M; iy++)
      for (int64_t ix = 0; ix < M; ix++) {
        const int64_t r = (iz * M + iy) * M + ix;
        P.rowptr[r + 1] = P.rowptr[r] + (hi[ix] - lo[ix] + 1) * (hi[iy] - lo[iy] + 1) * (hi[iz] - lo[iz] + 1);
      }
  P.nnz = P.rowptr[P.ndof];
  if (P.nnz > INT32_MAX) return "3d: pattern too large";
  P.col.resize(P.nnz);
  for (int64_t iz = 0; iz < M; iz++)
    for (int64_t iy = 0; iy < M; iy++)
      for (int64_t ix = 0; ix < M; ix++) {
        int64_t q = P.rowptr[(iz * M + iy) * M + ix];
        for (int64_t jz = lo[iz]; jz <= hi[iz]; jz++)
          for (int64_t jy = lo[iy]; jy <= hi[iy]; jy++)
            for (int64_t jx = lo[ix]; jx <= hi[ix]; jx++) P.col[q++] = (int32_t)((jz * M + jy) * M + jx);
      }
  // gather map: contributions counted, then filled in cube order (stable per slot)
  auto slot_of = [&](int32_t r, int32_t c) -> int64_t {
    const int32_t *b = P.col.data() + P.rowptr[r], *en = P.col.data() + P.rowptr[r + 1];
    return (int64_t)(std::lower_bound(b, en, c) - P.col.data());
  };
  P.map.ptr.assign(P.nnz + 1, 0);
  for (int64_t e = 0; e < nc3; e++)
    for (int k = 0; k < nb; k++)
      for (int l = 0; l < nb; l++) P.map.ptr[slot_of(P.dofs[e * nb + k], P.dofs[e * nb + l]) + 1]++;
  for (int64_t s = 0; s < P.nnz; s++) P.map.ptr[s + 1] += P.map.ptr[s];
  std::vector<int64_t> fill(P.map.ptr.begin(), P.map.ptr.end() - 1);
  P.map.idx.resize(P.map.ptr[P.nnz]);
  P.map.w.assign(P.map.ptr[P.nnz], 1.0);
  for (int64_t e = 0; e < nc3; e++)
    for (int k = 0; k < nb; k++)
      for (int l = 0; l < nb; l++)
        P.map.idx[fill[slot_of(P.dofs[e * nb + k], P.dofs[e * nb + l])]++] = (int32_t)(e * 2 * nb * nb + 2 * (k * nb + l));
  return "";
}

}  // namespace landau
