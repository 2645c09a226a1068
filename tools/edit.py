"""Tiny exact-match editing helper: replace(path, old, new) fails if `old` is not unique."""
def replace(path, old, new, count=1):
    s = open(path).read()
    n = s.count(old)
    if n != count:
        raise SystemExit(f"edit: {path}: expected {count} match(es), found {n}: {old[:80]!r}")
    open(path, "w").write(s.replace(old, new))
