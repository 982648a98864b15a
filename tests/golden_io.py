"""Loader for tests/golden/*.txt fixtures."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def load_golden(name: str) -> dict:
    """Parse a tests/golden/*.txt fixture: '# ...' comments, 'key: v v v' lines
    ('|' separators are ignored).  Integer lists come back as lists of int."""
    out = {}
    with open(os.path.join(ROOT, "tests", "golden", name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            k, v = line.split(":", 1)
            toks = [t for t in v.replace("|", " ").split() if t]
            vals = [int(t) for t in toks]
            out[k.strip()] = vals[0] if len(vals) == 1 and k.strip() not in ("flags", "col") else vals
    return out
