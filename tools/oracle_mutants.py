#!/usr/bin/env python
"""Mutation test of the oracle's CPU pins (test infrastructure; CPU only).

Each mutant is one plausible slip in oracle/frugal_oracle.c (a dropped term, an off-by-one,
a wrong operand).  It is compiled to a scratch library and the `-m "not gpu"` oracle pins
run against it (FRUGAL_ORACLE_LIB); a mutant must be KILLED (some pin fails).

    python tools/oracle_mutants.py            # all mutants
    python tools/oracle_mutants.py A B        # some
"""
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "frugal_oracle.c")

MUTANTS = {
    # VERDICT r1 mutant A: the first occurrence of every later 64-chunk is dropped
    "A_chunk_first_dropped": ("memcpy(chunk, gr + a[c0].p * d, d * sizeof(float));",
                              "if (c0 == i) memcpy(chunk, gr + a[c0].p * d, d * sizeof(float)); "
                              "else memset(chunk, 0, d * sizeof(float));"),
    # VERDICT r1 mutant B and its D+-1 siblings: age-out one step late / early
    "B_ageout_late": ("m->last_update <= s - 1 - o->c.age_out", "m->last_update <= s - 2 - o->c.age_out"),
    "B_ageout_early": ("m->last_update <= s - 1 - o->c.age_out", "m->last_update <= s - o->c.age_out"),
    "ageout_hot_rows_too": ("m->state == OR_INFP && !is_hot(o, m->key, s) &&", "m->state == OR_INFP &&"),
    "chunk_32": ("#define OR_CHUNK 64", "#define OR_CHUNK 32"),
    "chunk_256": ("#define OR_CHUNK 64", "#define OR_CHUNK 256"),
    "chunk_last_dropped": ("int64_t c1 = c0 + OR_CHUNK < e ? c0 + OR_CHUNK : e;",
                           "int64_t c1 = c0 + OR_CHUNK < e ? c0 + OR_CHUNK : e - 1;"),
    "adagrad_eps_inside_sqrt": ("float den = sqrtf(G[j]) + eps;", "float den = sqrtf(G[j] + eps);"),
    "adagrad_G_after": ("G[j] = G[j] + sq;\n                float num", "float num"),
    "sgd_sign": ("w[j] = w[j] - t;", "w[j] = w[j] + t;"),
    "next_access_window_short": ("for (int64_t t = u + 1; t <= hi; t++) if (any_read",
                                 "for (int64_t t = u + 1; t < hi; t++) if (any_read"),
    "next_access_from_u": ("for (int64_t t = u + 1; t <= hi; t++) if (any_read",
                           "for (int64_t t = u; t <= hi; t++) if (any_read"),
    "host_reader_ignores_hot": ("return !(g == owner(o, k) && is_hot(o, k, t));", "return 1;"),
    "adjust_wrong_step": ("int64_t t = s + L - 1;\n    if (t < o->S && t >= 1)", "int64_t t = s + L;\n    if (t < o->S && t >= 1)"),
    "urgent_as_deferred": ("if (pr == s) {", "if (pr == s + 1) {"),
    "glue_grad_no_x": ("gr[f * d + j] = c * ((S[j] - e[j]) + xb[j]);", "gr[f * d + j] = c * (S[j] - e[j]);"),
    "loss_not_mean": ("o->loss[s] = nb ? loss / (double)nb : 0.0;", "o->loss[s] = loss;"),
    "merge_first_rank_only": ("for (int64_t j = 0; j < d; j++) gk[j] = first ? P[j] : gk[j] + P[j];",
                              "for (int64_t j = 0; j < d; j++) gk[j] = first ? P[j] : gk[j];"),
    "flush_hot_rows_push_G": ("flush_row(o, i, cold);\n    }\n    /* (c)", "flush_row(o, i, 1);\n    }\n    /* (c)"),
    # not listed: dropping the final flush's G push of clean hot rows is an EQUIVALENT mutant
    # with a static cache (every read is followed by an update, so a hot row that was ever
    # updated is dirty at the end and goes out with w and G anyway)
}


def run(name, old, new, src):
    if old not in src:
        return "NOT APPLICABLE (pattern missing)"
    with tempfile.TemporaryDirectory() as td:
        c = os.path.join(td, "m.c")
        so = os.path.join(td, "libm.so")
        open(c, "w").write(src.replace(old, new, 1))
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
                               "-o", so, c, "-lm"])
        env = dict(os.environ, FRUGAL_ORACLE_LIB=so)
        r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-m", "not gpu", "-p", "no:cacheprovider",
                            "tests/test_oracle_pins.py", "tests/test_oracle_dyncache.py"],
                           cwd=ROOT, env=env, capture_output=True, text=True)
        if r.returncode == 0:
            return "SURVIVED"
        failed = [l for l in r.stdout.splitlines() if l.startswith("FAILED")]
        return "killed by " + (failed[0].split()[1] if failed else "error")


def main():
    src = open(SRC).read()
    names = sys.argv[1:] or list(MUTANTS)
    bad = 0
    for n in names:
        key = next(k for k in MUTANTS if k == n or k.startswith(n + "_") or k == n)
        res = run(key, *MUTANTS[key], src)
        bad += not res.startswith("killed")
        print(f"{key:28s} {res}", flush=True)
    print(f"{len(names) - bad}/{len(names)} mutants killed")
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main())
