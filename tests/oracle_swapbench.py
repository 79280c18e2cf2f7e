"""The configs[1] bench workload with an oracle mirror (test infrastructure).

bench.SwapBench drives the library; this subclass additionally mirrors every allocation in the
oracle's slab allocator (oracle/slab.py, O2: the library's handles must equal the oracle's, call by
call), places the input content with the oracle's own address function (oracle/kv.py `addr`, not the
library's block table), and afterwards replays the recorded round trips on the oracle's chunk-label
image of both pools (O5/O6) to check EVERY chunk of the device pool (batch, resident requests,
never-allocated poison) and every host chunk the oracle says was written."""
from __future__ import annotations

import numpy as np

import bench
from oracle import kv as OK
from oracle.shape import KVShape
from oracle.slab import SlabPool

GIB = bench.GIB


class OracleSwapBench(bench.SwapBench):
    def __init__(self, *a, **kw):
        super().__init__(*a, **kw)
        self.osh = KVShape(*self.sht)
        self.dg = OK.PoolGeom(self.cfg.device_kv_bytes, GIB, self.aeg.LAYER_MAJOR)
        self.hg = OK.PoolGeom(self.cfg.host_kv_bytes, GIB, self.aeg.LAYER_MAJOR)
        self.od, self.oh = SlabPool(self.dg.nbytes, GIB), SlabPool(self.hg.nbytes, GIB)

    def alloc_both(self, pool, n):
        c = self.ctx.kv_alloc(pool, self.sht, n)
        o = (self.od if pool == 0 else self.oh).alloc(self.osh, n)
        assert [(s, j) for _, s, j in map(self.aeg.decode_block, c)] == list(o), "allocator diverged from oracle"
        return c, o

    def setup(self):
        from aeg_inputs import dev as D
        gi, sh = self.gi, self.osh
        # never-allocated bytes carry their offset-keyed poison: the label image starts as poison
        D.fill_region(self.dbase, self.dg.nbytes, self.seed, gi.poison_key(gi.TAG_NEVER, 0))
        cells = self.dg.nbytes // self.Cl
        self.lab = (np.uint64(gi.poison_key(gi.TAG_NEVER, 0))
                    + np.arange(cells, dtype=np.uint64) * np.uint64(self.Cl // 8))
        self.hlab = np.zeros(self.hg.nbytes // self.Cl, dtype=np.uint64)   # 0 = unknown content
        live = []
        for op, v in gi.churn_ops(2, capacity_blocks=self.churn_slabs * self.k, hi_blocks=96):
            if op == "alloc":
                live.append(self.alloc_both(0, v))
            elif live[v] is not None:
                self.ctx.kv_free(0, live[v][0])
                self.od.free(live[v][1])
                live[v] = None
        churn = [x for x in live if x is not None]
        offs, keys = [], []
        for q, (c, o) in enumerate(churn):
            for j, h in enumerate(o):
                for l in range(sh.L):
                    offs.append(OK.addr(self.dg, sh, h, l))
                    keys.append(gi.kv_key(2, q % 65536, j, l))
        self._fill_lab(offs, keys)
        self.churn = [c for c, _ in churn]
        self.churn_offs, self.churn_keys = np.asarray(offs, np.uint64), np.asarray(keys, np.uint64)
        self.src_c, self.src_o = self.alloc_both(0, self.n)
        offs, keys = [], []
        for (r, j), h in zip(self.labels, self.src_o):
            for l in range(sh.L):
                offs.append(OK.addr(self.dg, sh, h, l))
                keys.append(gi.kv_key(1, r, j, l))
        self._fill_lab(offs, keys)
        return self

    def _fill_lab(self, offs, keys):
        offs = np.asarray(offs, np.uint64)
        keys = np.asarray(keys, np.uint64)
        self._fill(offs, keys)
        self.lab[(offs // np.uint64(self.Cl)).astype(np.int64)] = keys

    def replay_and_verify(self):
        """Oracle replay of the recorded round trips; full device-pool check + written host chunks +
        sampled chunks against the NumPy generator."""
        from aeg_inputs import dev as D
        gi, aeg, sh = self.gi, self.aeg, self.osh
        src_o = self.src_o
        for hc, nd in self.ops:
            hco = self.oh.alloc(sh, self.n)
            ndo = self.od.alloc(sh, self.n)
            assert [(s, j) for _, s, j in map(aeg.decode_block, hc)] == list(hco), "host allocator diverged"
            assert [(s, j) for _, s, j in map(aeg.decode_block, nd)] == list(ndo), "device allocator diverged"
            xo = self.od.begin(src_o)
            self.od.free(src_o)
            yo = self.oh.begin(hco)
            self.oh.free(hco)
            self.hlab = OK.swap_out(self.lab, self.dg, self.hlab, self.hg, sh, src_o, hco, unit=self.Cl)
            self.lab = OK.swap_in(self.hlab, self.hg, self.lab, self.dg, sh, hco, ndo, unit=self.Cl)
            self.od.complete(xo)
            self.oh.complete(yo)
            src_o = ndo
        self.src_o = src_o
        cells = self.lab.size
        bad_total = self._verify(self.dbase, np.arange(cells, dtype=np.uint64) * np.uint64(self.Cl), self.lab)
        known = np.nonzero(self.hlab)[0]
        hbad = self._verify(self.hbase, known.astype(np.uint64) * np.uint64(self.Cl), self.hlab[known])
        rng = np.random.default_rng(7)
        sample_bad = 0
        batch_cells = [OK.addr(self.dg, sh, h, l) // self.Cl for h in self.src_o for l in (0, sh.L - 1)]
        for c in rng.choice(batch_cells, size=8, replace=False):
            got = D.read(self.dbase + int(c) * self.Cl, self.Cl)
            sample_bad += int((got != gi.region_bytes(self.seed, int(self.lab[c]), self.Cl)).sum())
        return {"device_chunks_checked": int(cells), "device_bad_words": int(bad_total),
                "host_chunks_checked": int(known.size), "host_bad_words": int(hbad),
                "numpy_sampled_chunks": 8, "numpy_sampled_bad_bytes": sample_bad,
                "ok": bad_total == 0 and hbad == 0 and sample_bad == 0}

    def replay_given_and_verify(self, ops):
        """Oracle replay of round trips whose placements the library chose (ops = [(src, hc, nd)]
        library handles, in host issue order) — for round trips issued back to back, where which
        reclaimed blocks an allocation gets depends on GPU progress.  Sequential replay in host
        order is the result rules ❷❸ must produce however the transfers overlapped.  Checks every
        chunk of the device pool and every host chunk written."""
        aeg, sh = self.aeg, self.osh
        dec = lambda bs: [(s, j) for _, s, j in map(aeg.decode_block, bs)]  # noqa: E731
        for src, hc, nd in ops:
            self.hlab = OK.swap_out(self.lab, self.dg, self.hlab, self.hg, sh, dec(src), dec(hc), unit=self.Cl)
            self.lab = OK.swap_in(self.hlab, self.hg, self.lab, self.dg, sh, dec(hc), dec(nd), unit=self.Cl)
        cells = self.lab.size
        bad_total = self._verify(self.dbase, np.arange(cells, dtype=np.uint64) * np.uint64(self.Cl), self.lab)
        known = np.nonzero(self.hlab)[0]
        hbad = self._verify(self.hbase, known.astype(np.uint64) * np.uint64(self.Cl), self.hlab[known])
        return {"device_chunks_checked": int(cells), "device_bad_words": int(bad_total),
                "host_chunks_checked": int(known.size), "host_bad_words": int(hbad),
                "ok": bad_total == 0 and hbad == 0}

