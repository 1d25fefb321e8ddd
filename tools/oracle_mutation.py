"""Mutation run over the oracle's pins.

Each mutation edits a scratch copy of oracle/oracle.c (the repo is not
touched), rebuilds it, and runs tests/test_oracle_pins.py against it.  A
mutation is "killed" when at least one pin fails.  Usage:
    python tools/oracle_mutation.py            # all mutations
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (name, exact text in oracle.c, replacement)
MUTATIONS = [
    ("jenkins constant 0x7ed55d16 -> 0x7ed55d17", "0x7ed55d16u", "0x7ed55d17u"),
    ("jenkins shift <<12 -> <<11", "(a << 12)", "(a << 11)"),
    ("jenkins shift >>19 -> >>18", "(a >> 19)", "(a >> 18)"),
    ("jenkins constant 0xb55a4f09 -> 0xb55a4f08", "0xb55a4f09u", "0xb55a4f08u"),
    ("secondary-table insert deleted",
     "else if (sec[ss] < 0) { sec[ss] = r; tabled++; progress++; }", ""),
    ("secondary slot from the primary hash (h % S)",
     "int64_t ss = (int64_t)(oracle_jenkins32(h) % (uint32_t)S);\n            if (prim[ps] < 0)",
     "int64_t ss = (int64_t)(h % (uint32_t)S);\n            if (prim[ps] < 0)"),
    ("primary table size P = 4 S", "P = 5 * S;", "P = 4 * S;"),
]


def run(name, old, new):
    tmp = tempfile.mkdtemp(prefix="omut")
    try:
        for d in ("oracle", "synth", "tests"):
            shutil.copytree(os.path.join(ROOT, d), os.path.join(tmp, d),
                            ignore=shutil.ignore_patterns("*.so", "__pycache__"))
        src = os.path.join(tmp, "oracle", "oracle.c")
        text = open(src).read()
        assert text.count(old) >= 1, "mutation site not found: " + name
        open(src, "w").write(text.replace(old, new, 1))
        res = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                              "tests/test_oracle_pins.py"], cwd=tmp, capture_output=True, text=True)
        tail = res.stdout.strip().splitlines()[-1] if res.stdout.strip() else res.stderr[-200:]
        failed = [l for l in res.stdout.splitlines() if l.startswith("FAILED")]
        return res.returncode != 0, tail, failed[:1]
    finally:
        shutil.rmtree(tmp, ignore_errors=True)


if __name__ == "__main__":
    ok = True
    for name, old, new in MUTATIONS:
        killed, tail, first = run(name, old, new)
        ok &= killed
        print("%-48s %s  %s %s" % (name, "KILLED" if killed else "SURVIVED", tail, first[0] if first else ""))
    sys.exit(0 if ok else 1)
