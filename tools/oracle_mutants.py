"""Mutation check of the oracle's Stage-2 pins.

Builds a scratch copy of the repo per mutant of oracle/oracle.c (each a plausible misreading
of Alg. 3, PAPER.md file lines 442-480), runs the oracle's -m "not gpu" reorder pins there and
reports which mutants survive.  usage: python tools/oracle_mutants.py [pytest targets...]
"""
import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MUTANTS = {
    "priority list ascending (L400 'pick the worst')":
        ("if (x->score != y->score) return x->score > y->score ? -1 : 1;",
         "if (x->score != y->score) return x->score < y->score ? -1 : 1;"),
    "priority ties by id descending":
        ("return (x->seg > y->seg) - (x->seg < y->seg);                  /* then id ascending */",
         "return (x->seg < y->seg) - (x->seg > y->seg);"),
    "est[t] += gt (line 17 sign)": ("w->est[t] -= pr.gt;", "w->est[t] += pr.gt;"),
    "target never leaves I (lines 18-19)": ("if (w->est[t] <= 0) w->inI[t] = 0;", ";"),
    "no primary break on est <= 0 (lines 20-22)":
        ("if (w->est[p] <= 0 || all_positions_used(w->used, p, M, n)) break; /* lines 20-22 */",
         "if (all_positions_used(w->used, p, M, n)) break;"),
    "est[p] -= gt (line 16 operand)":
        ("w->est[p] -= pr.gp;                             /* line 16 */",
         "w->est[p] -= pr.gt;                             /* line 16 */"),
    "targets in reverse priority order (line 10)":
        ("for (int64_t k = 0; k < ns; ++k) { /* line 10: targets in priority order */",
         "for (int64_t k = ns - 1; k >= 0; --k) { /* line 10: targets in priority order */"),
    "freshtop ties -> last pair": ("if (!best.found || g > best.g) {", "if (!best.found || g >= best.g) {"),
    "freshtop ties -> largest v":
        ("for (int64_t v = t * M; v < t * M + M && v < n; ++v) {",
         "for (int64_t v = t * M + M - 1; v >= t * M; --v) { if (v >= n) continue;"),
    "gain: wrong d sign in segment p": ("sp += (cp > N) - (cp + d > N);", "sp += (cp > N) - (cp - d > N);"),
    "single-entry branch accepts any gain (L402 'beneficial')":
        ("or_pair pr = freshtop(B, N, M, p, t, w->used, 1);", "or_pair pr = freshtop(B, N, M, p, t, w->used, 0);"),
    "single-entry branch: densest target (L402 'sparsest')":
        ("if (t < 0 || z < tn) { t = s; tn = z; }", "if (t < 0 || z > tn) { t = s; tn = z; }"),
    "single-entry branch: no stop on est <= 0":
        ("if (w->est[p] <= 0 || all_positions_used(w->used, p, M, n)) break;\n    }\n    if (npairs",
         "if (all_positions_used(w->used, p, M, n)) break;\n    }\n    if (npairs"),
}


def main():
    targets = sys.argv[1:] or ["tests/test_oracle_stage2_fixtures.py", "tests/test_oracle_reorder.py"]
    src = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    survivors = 0
    for name, (a, b) in MUTANTS.items():
        assert src.count(a) == 1, name
        with tempfile.TemporaryDirectory() as d:
            for sub in ("oracle", "tests", "paper_conf_ppopp_chensz0s25_b200"):
                shutil.copytree(os.path.join(ROOT, sub), os.path.join(d, sub),
                                ignore=shutil.ignore_patterns("*.so", "_build", "__pycache__"))
            shutil.copy(os.path.join(ROOT, "pytest.ini"), d)
            open(os.path.join(d, "oracle", "oracle.c"), "w").write(src.replace(a, b))
            r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider", *targets],
                               cwd=d, capture_output=True, text=True)
            last = r.stdout.strip().splitlines()[-1] if r.stdout.strip() else r.stderr[-200:]
            killed = r.returncode != 0
            survivors += not killed
            print("%-60s %s  (%s)" % (name, "killed" if killed else "SURVIVES", last), flush=True)
    print("survivors: %d of %d" % (survivors, len(MUTANTS)))
    return 1 if survivors else 0


if __name__ == "__main__":
    sys.exit(main())
