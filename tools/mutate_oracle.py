"""Mutation check for the oracle pins: apply one plausible mistake at a time to oracle/ and
confirm that `pytest tests/test_oracle_*.py` fails.  Usage: python tools/mutate_oracle.py"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MUTANTS = [
    ("oracle/kv.py", "return s * g.slab_bytes + l * k * Cl + j * Cl", "return s * g.slab_bytes + j * k * Cl + l * Cl"),
    ("oracle/kv.py", "return s * g.slab_bytes + j * L * Cl + l * Cl", "return s * g.slab_bytes + l * L * Cl + j * Cl"),
    ("oracle/kv.py", "d = ((l - l0) * n + i) * c\n            stage[d:d + c]", "d = (i * (l1 - l0) + (l - l0)) * c\n            stage[d:d + c]"),
    ("oracle/kv.py", "out[a:a + c] = stage[d:d + c]", "out[a:a + c] = stage[d:d + c][::-1]"),
    ("oracle/kv.py", "out = dst.copy()", "out = np.zeros_like(dst)"),
    ("oracle/shape.py", "return self.L * 2 * self.H * self.D * self.s", "return self.L * self.H * self.D * self.s"),
    ("oracle/shape.py", "return (((c * self.B + slot) * self.H + h) * self.D + d) * self.s", "return (((c * self.B + h) * self.H + slot) * self.D + d) * self.s"),
    ("oracle/slab.py", "if j not in self.owned[s] and (s, j) not in self.quarantine:", "if j not in self.owned[s]:"),
    ("oracle/slab.py", "for s in range(self.n_slabs):\n            if self.shape[s] is not None:", "for s in reversed(range(self.n_slabs)):\n            if self.shape[s] is not None:"),
    ("oracle/slab.py", "if busy:\n                self.quarantine[(s, j)] = busy", "if False:\n                self.quarantine[(s, j)] = busy"),
    ("oracle/slab.py", "                self.shape[s] = None\n", "                pass\n"),
    ("oracle/slab.py", "return self.slab_bytes // shape.block_bytes()", "return -(-self.slab_bytes // shape.block_bytes())"),
    ("oracle/weights.py", "return w[:, r * part:(r + 1) * part]", "return w[:, r:(r + 1) * part]"),
    ("oracle/weights.py", "for gi in range(groups)], axis=0)", "for gi in range(groups)][::-1], axis=0)"),
    ("oracle/weights.py", "p = align_up(p + n)", "p = p + n"),
    ("oracle/memmove.py", "out[dst:dst + n] = tmp", "out[dst:dst + n] = tmp[::-1]"),
    ("oracle/memmove.py", "tmp = buf[src:src + n].copy()", "tmp = buf[dst:dst + n].copy()"),
    ("oracle/weights.py", "if offs and offs[-1] + shards[-1].size > region_bytes:", "if offs and offs[-1] > region_bytes:"),
    ("oracle/weights.py", "if offs and offs[-1] + shards[-1].size > region_bytes:", "if offs and offs[-1] + shards[-1].size >= region_bytes:"),
    ("oracle/slab.py", "return 0.0 if peak == 0 else (assigned - used) / peak", "return 0.0 if assigned == 0 else (assigned - used) / assigned"),
    ("oracle/slab.py", "self.peak_assigned = max(self.peak_assigned, sum(v[0] for v in per.values()) * self.slab_bytes)", "self.peak_assigned = sum(v[0] for v in per.values()) * self.slab_bytes"),
    ("oracle/rules.py", "pending.setdefault(e[1], set()).add(c)", "pass"),
    ("oracle/rules.py", "captured[e[2]] = tail.get(e[1])", "captured[e[2]] = len(ops) - 1 if ops else None"),
    ("oracle/rules.py", "            p.update(synced)\n", "            pass\n"),
    ("oracle/rules.py", "            a |= anc[q]\n", "            pass\n"),
    ("oracle/rules.py", "            if w is not None and w not in anc[i]:\n                rule", "            if False:\n                rule"),
    ("oracle/rules.py", "for r in reads_since.get(c, ()):", "for r in ():"),
    ("oracle/rules.py", "rule = \"❶\" if kind == \"use\" else \"❷\"", "rule = \"❷\""),
    ("oracle/kv.py", "out = dst.copy()", "out = dst"),
    ("oracle/kv.py", "    out = pool.copy()\n    n, c = len(handles), _c(sh, unit)", "    out = pool\n    n, c = len(handles), _c(sh, unit)"),
    ("oracle/weights.py", "if rows % (groups * tp):", "if rows % tp:"),
    ("oracle/weights.py", "if cols % tp or groups != 1:", "if cols % tp:"),
    ("oracle/weights.py", "        dst = dst.copy()\n", "        pass\n"),
    ("oracle/weights.py", "        offs.append(p)\n        p = align_up(p + n)", "        p = align_up(p + n)\n        offs.append(p)"),
    ("oracle/kv.py", "    k = g.slab_bytes // sh.block_bytes()\n    assert", "    k = g.slab_bytes // sh.chunk_bytes()\n    assert"),
    ("oracle/kv.py", "    stage = np.empty((l1 - l0) * n * c, dtype=pool.dtype)\n    for l in range(l0, l1):",
     "    stage = np.empty((l1 - l0) * n * c, dtype=pool.dtype)\n    for l in range(l0, max(l0, l1 - 1)):"),
    ("oracle/slab.py", "        self.reclaim()                              # reading 9", "        pass  # reading 9"),
    ("oracle/slab.py", "if self.shape[s] is not None and not self.owned[s] and not any(q[0] == s for q in self.quarantine):",
     "if self.shape[s] is not None and not self.owned[s]:"),
    ("oracle/slab.py", "if xs <= self.done]", "if xs & self.done]"),
    ("oracle/slab.py", "if j not in self.owned[s] or (s, j) in seen:", "if j not in self.owned[s]:"),
    ("oracle/slab.py", "if x not in self.done and b in blocks}", "if b in blocks}"),
    ("oracle/slab.py", "if n < 0 or self.k(shape) == 0:", "if n <= 0 or self.k(shape) == 0:"),
    ("oracle/slab.py", "peak = self.peak_assigned_shape.get(shape, 0)", "peak = self.peak_assigned"),
]


def run_one(path, old, new):
    """Apply one mutant in a private copy of oracle/ + tests/ and run the oracle pins there."""
    with tempfile.TemporaryDirectory() as d:
        for sub in ("oracle", "tests", "aeg_inputs"):
            shutil.copytree(os.path.join(ROOT, sub), os.path.join(d, sub),
                            ignore=shutil.ignore_patterns("__pycache__", "*.so"))
        f = os.path.join(d, path)
        src = open(f).read()
        assert old in src, (path, old)
        open(f, "w").write(src.replace(old, new, 1))
        r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider",
                            "tests/test_oracle_shape.py", "tests/test_oracle_slab.py", "tests/test_oracle_kv.py",
                            "tests/test_oracle_weights.py", "tests/test_oracle_rules.py", "tests/test_oracle_memmove.py"],
                           cwd=d, capture_output=True, text=True)
        return r.returncode != 0


def main(jobs=None):
    import concurrent.futures as cf
    jobs = jobs or max(1, min(16, os.cpu_count() or 1))
    with cf.ThreadPoolExecutor(max_workers=jobs) as ex:
        killed = list(ex.map(lambda m: run_one(*m), MUTANTS))
    survived = []
    for (path, _, new), k in zip(MUTANTS, killed):
        print(f"{'killed' if k else 'SURVIVED':9s} {path}: {new[:70]!r}")
        if not k:
            survived.append((path, new))
    print(f"{len(MUTANTS) - len(survived)}/{len(MUTANTS)} mutants killed")
    return 1 if survived else 0


if __name__ == "__main__":
    sys.exit(main(int(sys.argv[1]) if len(sys.argv) > 1 else None))
