"""A CPU replica of the staged Algorithm-2 construction (the builder protocol of
dist.build_distributed: info / group_rows / phase1 / export_rows / import_rows /
round_search / round_apply / finish) -- TEST INFRASTRUCTURE.

It restates Algorithm 2 with numpy rows and Python sorts, using the
oracle's O2 search (pinned by Example 2, brute force and invariants) as its
search step, so the gloo tests can run the multi-rank orchestration on CPU and
compare the result with oracle.alg2 bit for bit."""
import numpy as np
import torch

import oracle


class PyStagedBuild:
    def __init__(self, X, d_min, d_max, group_size, l_build, l_local=0, metric="l2"):
        self.X = np.ascontiguousarray(X, np.float32)
        self.n = len(X)
        self.d_min, self.d_max, self.S = d_min, d_max, group_size
        self.G = (self.n + group_size - 1) // group_size
        self.l_build, self.l_local = l_build, (l_local or l_build)
        self.metric = metric
        self.ids = np.full((self.n, d_max), -1, np.int32)
        self.dists = np.full((self.n, d_max), np.inf, np.float32)
        self.pids = np.full((self.n, d_min), -1, np.int32)
        self.pdists = np.full((self.n, d_min), np.inf, np.float32)
        self.searches = 0

    # -- protocol
    def info(self):
        return self.S, self.G, self.d_min, self.d_max

    def group_rows(self, g0, g1):
        return min(g0 * self.S, self.n), min(g1 * self.S, self.n)

    def _row(self, v):
        return [(float(d), int(i)) for d, i in zip(self.dists[v], self.ids[v]) if i >= 0]

    def _set_row(self, v, row):
        row = row[:self.d_max]
        self.ids[v] = -1
        self.dists[v] = np.inf
        for j, (d, i) in enumerate(row):
            self.ids[v, j], self.dists[v, j] = i, d

    def _search(self, v, k, l, entry):
        self.searches += 1
        i, d = oracle.search(self.ids, self.X, self.X[v][None], k, l, entry=entry,
                             metric=self.metric)
        return [(float(dd), int(ii)) for dd, ii in zip(d[0], i[0]) if ii >= 0]

    def phase1(self, g0, g1):
        """Alg. 2 lines 2-8: sequential insertion into each local graph."""
        for g in range(g0, g1):
            lo, hi = self.group_rows(g, g + 1)
            for v in range(lo, hi):
                F = [] if v == lo else self._search(v, self.d_min, self.l_local, lo)[:self.d_min]
                self._set_row(v, F)
                self.pids[v] = -1
                self.pdists[v] = np.inf
                for j, (d, u) in enumerate(F):
                    self.pids[v, j], self.pdists[v, j] = u, d
                for d, u in F:
                    self._set_row(u, sorted(self._row(u) + [(d, v)]))

    def export_rows(self, v0, v1):
        return tuple(torch.from_numpy(a[v0:v1].copy())
                     for a in (self.ids, self.dists, self.pids, self.pdists))

    def import_rows(self, v0, v1, rows):
        for a, t in zip((self.ids, self.dists, self.pids, self.pdists), rows):
            a[v0:v1] = t.cpu().numpy()

    def round_search(self, i, v0, v1):
        """Lines 10-17 for [v0, v1) of P_i: F = first d_min of Search(G_0, v) u v.N'."""
        fi = np.full((v1 - v0, self.d_min), -1, np.int32)
        fd = np.full((v1 - v0, self.d_min), np.inf, np.float32)
        for v in range(v0, v1):
            S = self._search(v, self.d_min, self.l_build, 0)[:self.d_min]
            Np = [(float(d), int(u)) for d, u in zip(self.pdists[v], self.pids[v]) if u >= 0]
            for j, (d, u) in enumerate(sorted(S + Np)[:self.d_min]):
                fi[v - v0, j], fd[v - v0, j] = u, d
        return torch.from_numpy(fi), torch.from_numpy(fd)

    def round_apply(self, i, f_ids, f_dists):
        """Rows of P_i <- F (R-C15); E sorted by (u, dist, v) (R-C17); per u the
        first d_max of merge(u.N, segment) (lines 19-22)."""
        lo, hi = self.group_rows(i, i + 1)
        fi, fd = f_ids.cpu().numpy(), f_dists.cpu().numpy()
        E = []
        for v in range(lo, hi):
            F = [(float(d), int(u)) for d, u in zip(fd[v - lo], fi[v - lo]) if u >= 0]
            self._set_row(v, F)
            E += [(u, d, v) for d, u in F]
        E.sort()
        for u in sorted({e[0] for e in E}):
            seg = [(d, v) for uu, d, v in E if uu == u]
            self._set_row(u, sorted(self._row(u) + seg))

    def finish(self):
        return self.ids.copy()
