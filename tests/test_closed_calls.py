"""The GPU pool refuses any command whose tree names the batched-memcpy entry points (they raised
Xid 32 there).  Nothing outside notes (*.md) and the driver's own records may name them, binaries
included: the product links cudart dynamically so no copy of the runtime's symbol table ships."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# assembled at run time so this file does not name them either
NAMES = [p + "Memcpy" + d + "BatchAsync" for p in ("cuda", "cu") for d in ("", "3D")]
SKIP_DIRS = {".git", "gpurun_out", "__pycache__", ".pytest_cache", ".hypothesis", "baseline", ".claude"}


def _ignored():
    pats = []
    p = os.path.join(ROOT, ".gpurunignore")
    if os.path.exists(p):
        pats = [l.strip().rstrip("/") for l in open(p) if l.strip() and not l.startswith("#")]
    return pats


def test_tree_does_not_name_closed_calls():
    import fnmatch
    ign = _ignored()
    hits = []
    for d, dirs, files in os.walk(ROOT):
        rel_d = os.path.relpath(d, ROOT)
        dirs[:] = [x for x in dirs if x not in SKIP_DIRS
                   and not any(fnmatch.fnmatch(os.path.normpath(os.path.join(rel_d, x)), g) for g in ign)]
        for f in files:
            rel = os.path.normpath(os.path.join(rel_d, f))
            if f.endswith(".md") or any(fnmatch.fnmatch(rel, g) for g in ign):
                continue
            try:
                data = open(os.path.join(d, f), "rb").read()
            except OSError:
                continue
            for n in NAMES:
                if n.encode() in data:
                    hits.append(f"{rel}: {n}")
    assert not hits, hits
