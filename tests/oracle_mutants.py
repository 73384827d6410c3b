"""Mutation check of the oracle's pins (test infrastructure, run by hand on
CPU; not collected by pytest):

    python tests/oracle_mutants.py [--jobs 4] [--out profiles/oracle_mutants.txt]

Each mutant is one plausible mistake written into a copy of the repository
(a dropped term, a flipped sign or comparison, a transposed operand, an
off-by-one, a wrong digit order ...) in oracle/abacus_oracle.c, oracle/train.py,
oracle/__init__.py or oracle/brute.py.  The pin files (PINS: the oracle
against worked examples, closed forms, brute force, exact rationals and known
answers -- not against the product) run against the mutated oracle; a mutant
is KILLED when some pin fails.  The
unmutated copy must pass (control).  A surviving mutant names a gap in the
pins -- or an equivalent mutant, which the table says.  Nothing here touches
the CUDA path; the copies live under /tmp."""
import argparse
import os
import shutil
import subprocess
import sys
import tempfile
import time
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
C = "oracle/abacus_oracle.c"
TR = "oracle/train.py"
PY = "oracle/__init__.py"
BR = "oracle/brute.py"

# (name, file, find, replace, occurrence) -- occurrence None: the text must be unique
MUTANTS = [
    ("Eq.3: in-flight prediction added instead of subtracted", C,
     "return t_h - inflight_pred_ms;", "return t_h + inflight_pred_ms;", None),
    ("Eq.2: elapsed time sign flipped", C,
     "double t_h = qos_ms - (now_ms - t_start_ms);", "double t_h = qos_ms - (t_start_ms - now_ms);", None),
    ("order: descending headroom", C,
     "while (j >= 0 && (h[order[j]] > h[v] ||", "while (j >= 0 && (h[order[j]] < h[v] ||", None),
    ("order: ties broken by descending model id (c10)", C,
     "(h[order[j]] == h[v] && model_id[order[j]] > model_id[v]))", "(h[order[j]] == h[v] && model_id[order[j]] < model_id[v]))", None),
    ("Fig.8: multi-hot bit at model id, not id - 1", C,
     "x[tmp[p].model_id - 1] = 1;", "x[tmp[p].model_id % n_models] = 1;", None),
    ("Fig.8: ops and ope swapped", C,
     "x[n_models + 4 * p + 0] = (int16_t)tmp[p].ops;", "x[n_models + 4 * p + 0] = (int16_t)tmp[p].ope;", None),
    ("Fig.8: slots not sorted by model id", C,
     "while (j >= 0 && tmp[j].model_id > v.model_id)", "while (0 && j >= 0 && tmp[j].model_id > v.model_id)", None),
    ("Fig.8: bs and seqlen swapped", C,
     "x[n_models + 4 * p + 2] = (int16_t)tmp[p].bs;", "x[n_models + 4 * p + 2] = (int16_t)tmp[p].seqlen;", None),
    ("MLP: layer-2 ReLU dropped", C, "h2[i] = s > 0.0 ? s : 0.0;", "h2[i] = s;", 0),
    ("MLP: b3 dropped", C, "s += (double)b3[i];", "s += 0.0;", None),
    ("MLP: W2 transposed", C, "s += (double)W2[i * ORC_H + j] * h1[j];", "s += (double)W2[j * ORC_H + i] * h1[j];", None),
    ("MLP: b4 dropped", C, "return y + (double)b4[0];", "return y;", None),
    ("MLP: W1 read column-major", C, "s += (double)W1[i * d + j] * (double)x[j];",
     "s += (double)W1[(j * ORC_H + i) % (ORC_H * d)] * (double)x[j];", None),
    ("MLP: output ReLU added", C, "return y + (double)b4[0];", "return fmax(y + (double)b4[0], 0.0);", None),
    ("key: sum_n without the +1 (c12)", C, "uint64_t key = ((uint64_t)(sum_n + 1) << 40) | t;",
     "uint64_t key = ((uint64_t)(sum_n) << 40) | t;", None),
    ("mask: y < H instead of y <= H (c11)", C, "if (y <= st->H) {", "if (y < st->H) {", None),
    ("digits: absent digit off by one", C, "if (s->allow_absent) st->ope[j] = dgt == 0 ? 0 : s->end_lo + dgt - 1;",
     "if (s->allow_absent) st->ope[j] = dgt == 0 ? 0 : s->end_lo + dgt;", None),
    ("n = ope - ops without the +1 (c7)", C, "sum_n += st->ope[j] - st->g[j].start_op + 1;",
     "sum_n += st->ope[j] - st->g[j].start_op;", None),
    ("grid size ignores the absent option", C,
     "        if (g[j].end_hi < g[j].end_lo) return 0;\n        T *= (uint64_t)(g[j].allow_absent + g[j].end_hi - g[j].end_lo + 1);",
     "        if (g[j].end_hi < g[j].end_lo) return 0;\n        T *= (uint64_t)(g[j].end_hi - g[j].end_lo + 1);", None),
    ("a2: critical query not fully included", C, "g[j].end_lo = j == 0 ? Lm : qq->next_op;",
     "g[j].end_lo = qq->next_op;", 0),
    ("a2: critical query may be absent", C, "g[j].allow_absent = j == 0 ? 0 : 1;", "g[j].allow_absent = 1;", 0),
    ("H kept in double (not the fp32 the GPU sees)", C, "double H = (double)(float)h[order[0]];          /* the fp32",
     "double H = h[order[0]];          /* the fp32", None),
    ("drop: y(0) < H instead of <=", C, "if (!(out->pred_critical_only_ms <= H)) {",
     "if (!(out->pred_critical_only_ms < H)) {", None),
    ("CHAIN: earlier slots at their start op, not full", C, "if (i < j) ope[i] = g[i].end_hi;",
     "if (i < j) ope[i] = g[i].start_op;", 0),
    ("CHAIN: partial slot off by one", C,
     "else if (i == j) ope[i] = j == 0 ? g[0].end_hi : g[i].start_op + dd - 1;",
     "else if (i == j) ope[i] = j == 0 ? g[0].end_hi : g[i].start_op + dd;", None),
    ("AUTO: GRID only below the budget (>= instead of >)", C,
     "int32_t use_chain = space == 1 || (space == 2 && T > budget);",
     "int32_t use_chain = space == 1 || (space == 2 && T >= budget);", None),
    ("decode: digits read most-significant first", C,
     "        for (int32_t j = k - 1; j >= 0; j--) {\n            uint64_t radix",
     "        for (int32_t j = 0; j < k; j++) {\n            uint64_t radix", None),
    ("y(0) taken at index 1", C, "if (t == 0) r->y0 = y;", "if (t == 1) r->y0 = y;", None),
    ("acceptance window absolute, not relative (c18)", C, "double tol = st->eps * fabs(st->H);",
     "double tol = st->eps;", None),
    ("bf16 rounding truncates", C, "double r = nearbyint(scaled);", "double r = trunc(scaled);", None),
    ("bf16 keeps 7 significant bits", C, "double scaled = ldexp(m, 8);", "double scaled = ldexp(m, 7);", None),
    ("m-way: lo restarts at the critical query", C, "lo = probes[last];", "lo = probes[0];", None),
    ("m-way: probes spaced by ways, not ways + 1", C,
     "uint64_t v = lo + (span * (uint64_t)i) / (uint64_t)(ways + 1);",
     "uint64_t v = lo + (span * (uint64_t)i) / (uint64_t)ways;", None),
    ("m-way: lo moves to the first fitting probe", C, "if (f[i]) lf = i;", "if (f[i] && lf < 0) lf = i;", None),
    ("hash: index not mixed into the row hash", C, "r->hash += orc_splitmix64(t ^ orc_fnv1a64(x, st->d));",
     "r->hash += orc_splitmix64(orc_fnv1a64(x, st->d));", None),
    ("hash: SplitMix64 shift constant", C, "z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;",
     "z = (z ^ (z >> 28)) * 0x94D049BB133111EBULL;", None),
    ("hash: FNV bytes in big-endian order", C, "h ^= b0; h *= 0x100000001b3ULL;\n        h ^= b1;",
     "h ^= b1; h *= 0x100000001b3ULL;\n        h ^= b0;", None),
    ("shell: bound off by one", C, "if (psum + n_j + st->rest_max[j + 1] < st->nsum_min) {",
     "if (psum + n_j + st->rest_max[j + 1] <= st->nsum_min) {", None),
    ("train: loss gradient sign", TR, "g = 2.0 * r / t / B ", "g = -2.0 * r / t / B ", None),
    ("train: ReLU mask of layer 2 from z3", TR, "d2 = (d3 @ W3) * (z2 > 0)", "d2 = (d3 @ W3) * (z3 > 0)", None),
    ("train: W2 gradient transposed", TR, "gW2 = d2.T @ a1", "gW2 = (d2.T @ a1).T", None),
    ("train: Adam without bias correction", TR, "mh = self.m / (1.0 - self.b1 ** self.t)", "mh = self.m", None),
    ("train: Adam eps inside the sqrt", TR, "(np.sqrt(vh) + self.eps)", "np.sqrt(vh + self.eps)", None),
    ("train: MAPE divides by the prediction", TR, "np.abs(y_pred - y_true) / y_true", "np.abs(y_pred - y_true) / y_pred", None),
    ("what-if: variant as the least significant digit", PY,
     "lift = lambda key: ((key >> 40) << 40) | (v * T + (key & ((1 << 40) - 1))) if key else 0",
     "lift = lambda key: ((key >> 40) << 40) | ((key & ((1 << 40) - 1)) * len(variants) + v) if key else 0", None),
    ("what-if: first variant wins ties", PY, "if r.best_key and lift(r.best_key) > best[0]:",
     "if r.best_key and (lift(r.best_key) >> 40) > (best[0] >> 40):", None),
    ("brute: absent digit last instead of first", BR, None, None, None),
    ("Eq.3: in-flight prediction subtracted from the first query only (c15)", C,
     "h[i] = orc_headroom(q[i].qos_ms, q[i].t_start_ms, now_ms, inflight_ms);",
     "h[i] = orc_headroom(q[i].qos_ms, q[i].t_start_ms, now_ms, i == 0 ? inflight_ms : 0.0);", 0),
    ("bf16 emulation: layer-1 activations not rounded", C, "h1[i] = RA(s > 0.0 ? s : 0.0);",
     "h1[i] = (s > 0.0 ? s : 0.0);", None),
    ("bf16 emulation: biases rounded under the weight flag", C,
     "#define RB(v) ((flags & 2) ?", "#define RB(v) ((flags & 1) ?", None),
    ("encode_groups: unused slots kept", C, "if (groups[g * kmax + j].model_id != 0) s[n++]",
     "if (groups[g * kmax + j].model_id >= 0) s[n++]", None),
    ("sweep range: shard starts one index late", C, "if (st->counter >= st->first && st->counter < st->last) orc_visit(st);",
     "if (st->counter > st->first && st->counter < st->last) orc_visit(st);", None),
    ("CHAIN: block length without the +1", C, "int32_t R = j == 0 ? 1 : g[j].end_hi - g[j].start_op + 1;",
     "int32_t R = j == 0 ? 1 : g[j].end_hi - g[j].start_op;", None),
    ("m-way: never drops", C, "if (!fit[0]) {", "if (0 && !fit[0]) {", None),
]


def load_brute_mutant(src):
    """brute.slot_choices: the absent option moved from digit 0 to the end."""
    a = "return ch + list(range(s.end_lo, s.end_hi + 1))"
    if a in src:
        return src.replace(a, "return list(range(s.end_lo, s.end_hi + 1)) + ch")
    raise RuntimeError("brute mutant: pattern not found")


def make_copy(dst):
    ign = shutil.ignore_patterns(".git", "gpurun_out", "exp", "profiles", "__pycache__", "liboracle.so",
                                 ".pytest_cache", "*.ncu-rep")
    shutil.copytree(ROOT, dst, ignore=ign)


def apply(dst, m):
    name, f, find, repl, occ = m
    p = os.path.join(dst, f)
    src = open(p).read()
    if f == BR:
        out = load_brute_mutant(src)
    else:
        n = src.count(find)
        if occ is None and n != 1:
            raise RuntimeError("%s: pattern occurs %d times" % (name, n))
        if occ is not None and n <= occ:
            raise RuntimeError("%s: occurrence %d of %d" % (name, occ, n))
        i = -1
        for _ in range((occ or 0) + 1):
            i = src.index(find, i + 1)
        out = src[:i] + repl + src[i + len(find):]
    open(p, "w").write(out)


# the pins proper: checks of the oracle against the paper and the mathematics
# (worked examples, closed forms, brute force, exact rationals, known answers);
# the other CPU tests compare the product's host code with the oracle and do
# not count as pins
PINS = ["tests/test_oracle_pins.py", "tests/test_oracle_train.py", "tests/test_controller.py"]


def run_suite(dst, timeout, tests):
    t0 = time.time()
    try:
        p = subprocess.run([sys.executable, "-m", "pytest", *tests, "-x", "-q", "-m", "not gpu",
                            "-p", "no:cacheprovider"], cwd=dst, capture_output=True, text=True, timeout=timeout)
        rc, out = p.returncode, p.stdout
    except subprocess.TimeoutExpired:
        rc, out = -9, "timeout"
    first_fail = ""
    for line in out.splitlines():
        if line.startswith("FAILED") or line.startswith("ERROR"):
            first_fail = line.split(" - ")[0].replace("FAILED ", "").replace("ERROR ", "")
            break
    return rc, first_fail, time.time() - t0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--jobs", type=int, default=4)
    ap.add_argument("--out", default=None)
    ap.add_argument("--timeout", type=int, default=900)
    ap.add_argument("--only", type=int, nargs="*")
    ap.add_argument("--all-cpu-tests", action="store_true",
                    help="run the whole CPU suite per mutant instead of the pin files only")
    a = ap.parse_args()
    base = tempfile.mkdtemp(prefix="oracle_mut_")
    todo = [(i, m) for i, m in enumerate(MUTANTS) if not a.only or i in a.only]

    def one(item):
        i, m = item
        dst = os.path.join(base, "m%02d" % i if i >= 0 else "control")
        make_copy(dst)
        if m is not None:
            apply(dst, m)
        rc, ff, dt = run_suite(dst, a.timeout, ["tests"] if a.all_cpu_tests else PINS)
        shutil.rmtree(dst, ignore_errors=True)
        return i, m, rc, ff, dt

    lines = []
    _, _, rc, ff, dt = one((-1, None))
    lines.append("control (unmutated copy): %s (%.0f s)" % ("PASS" if rc == 0 else "FAIL rc=%d %s" % (rc, ff), dt))
    print(lines[-1], flush=True)
    if rc != 0:
        sys.exit(1)
    killed = 0
    with ThreadPoolExecutor(a.jobs) as ex:
        for i, m, rc, ff, dt in ex.map(one, todo):
            ok = rc != 0
            killed += ok
            lines.append("%2d %-8s %-55s %s" % (i, "KILLED" if ok else "SURVIVED", m[0],
                                                 ("by " + ff) if ok else "(suite green)"))
            print(lines[-1], flush=True)
    lines.append("killed %d of %d mutants" % (killed, len(todo)))
    print(lines[-1])
    shutil.rmtree(base, ignore_errors=True)
    if a.out:
        with open(a.out, "w") as f:
            f.write("# python tests/oracle_mutants.py --jobs %d%s  (%s against each mutated oracle)\n"
                    % (a.jobs, " --all-cpu-tests" if a.all_cpu_tests else "",
                       "the whole CPU suite" if a.all_cpu_tests else "the pin files " + " ".join(PINS)))
            f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
