"""Mutation check of the oracle's pins.

Each mutant is one plausible mistake in oracle/fastt_oracle.c (a dropped
term, a wrong sign / index / tie-break, a transposed rule).  For each, a
mutated copy is written to /tmp, built by oracle.build() through
FASTT_ORACLE_SRC, and the CPU pin suites are run against it; a mutant is
"killed" when at least one pin fails.  Usage:

    python tools/oracle_mutants.py [name ...]   # prints a table, exit 1 if any survives
"""
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "fastt_oracle.c")
PINS = ["tests/test_oracle_pins.py", "tests/test_oracle_alg2.py", "tests/test_oracle_n3.py"]

# name -> (paper passage / reading, exact text, replacement, occurrence index or None for unique)
MUTANTS = {
    "alg2_break_to_continue": ("Alg. 2 line 12, P:802 / R15",
                               "      if (bg) { fo_graph_free(bg); fo_result_free(&br); }\n      break;",
                               "      if (bg) { fo_graph_free(bg); fo_result_free(&br); }\n      continue;", 0),
    "cp_sort_ascending": ("Alg. 2 line 5, P:777 / R15", "if (cy > cx || (cy == cx && y < x)) break;",
                          "if (cy < cx || (cy == cx && y < x)) break;", None),
    "r9_truncated_average": ("P:600-609 / R9", "(__int128)S[d] * m[best] < (__int128)S[best] * m[d]",
                             "S[d] / m[d] < S[best] / m[best]", None),
    "priority_id_tiebreak_flipped": ("R2, R3", "  return a < b;\n}", "  return a > b;\n}", None),
    "eft_argmin_le": ("Alg. 1 lines 12-19, R3", "if (eft < best) { best = eft;", "if (eft <= best) { best = eft;", None),
    "est_drops_comm": ("P:571-574, R6", "int64_t t_ = r->finish[m_] + fo_comm(g, g->pred_bytes[e_], r->place[m_], dev);",
                       "int64_t t_ = r->finish[m_];", None),
    "rank_drops_w": ("P:539-554", "rank[i] = fo_w(g, pin, dset, i) + best;", "rank[i] = best;", None),
    "rank_drops_c": ("P:539-554, R5", "int64_t v = fo_c(g, pin, dset, i, j, g->succ_bytes[e]) + rank[j];",
                     "int64_t v = rank[j];", None),
    "w_min_not_max": ("P:543-544, R5", "if (g->cost[(int64_t)i * g->G + d] > mx) mx = g->cost[(int64_t)i * g->G + d];",
                      "if (d == 0 || g->cost[(int64_t)i * g->G + d] < mx) mx = g->cost[(int64_t)i * g->G + d];", None),
    "subop_cost_floor": ("R13", "ceil_div(g->cost[(int64_t)op * G + d], n)", "g->cost[(int64_t)op * G + d] / n", None),
    "partition_extra_to_last": ("R13", "return b / n + (k < b % n ? 1 : 0);", "return b / n + (k >= n - b % n ? 1 : 0);",
                                None),
    "batch_split_cuts_params": ("R13", "return dim == FO_DIM_BATCH ? !p : p;", "return dim == FO_DIM_BATCH ? p : !p;",
                                None),
    "cp_walk_lowest_rank": ("P:595-598, R7", "if (nxt < 0 || fo_higher(rank, j, nxt)) nxt = j;",
                            "if (nxt < 0 || fo_higher(rank, nxt, j)) nxt = j;", None),
    "cp_reservation_ignored": ("R8, R9", "if (used[d] + reserved[d] + mi > g->cap[d]) continue;",
                               "if (used[d] + mi > g->cap[d]) continue;", None),
    "cp_prefix_not_longest": ("P:600-609, R9", "while (k + m[d] < nf && msum + g->mem[fr[k + m[d]]] <= g->cap[d]) {",
                              "while (k + m[d] < nf && m[d] < 1 && msum + g->mem[fr[k + m[d]]] <= g->cap[d]) {", None),
    "r21_op_dev_draws_swapped": ("R21", "    uint64_t xo = fo_splitmix64(&st);\n    int32_t idx",
                                 "    uint64_t xd0 = fo_splitmix64(&st); (void)xd0;\n    uint64_t xo = fo_splitmix64(&st);\n    int32_t idx",
                                 None),
    "order_a_by_dequeue": ("Alg. 1 line 23, R17", "while (pos > 0 && r->start[r->order[pos - 1]] > r->start[i]) {",
                           "while (0) {", None),
    "comm_floor": ("R10", "return g->alpha[k] + (num + 999999) / 1000000;", "return g->alpha[k] + num / 1000000;", None),
    "insert_accepts_zero_len_slot": ("R1i", "    if (b > a) {\n      int64_t t = a > r ? a : r;",
                                     "    if (b >= a) {\n      int64_t t = a > r ? a : r;", None),
    "bi_accepts_ties": ("R23 (N2)", "if (!bg || bft >= ft_old) {", "if (!bg || bft > ft_old) {", None),
    "bi_tie_last_wins": ("R23 (N2)", "          if (r.status == FO_CAND_OK && r.makespan < bft) {\n            if (bg) { fo_graph_free(bg); fo_result_free(&br); }\n            bg = sv; br = r; bft = r.makespan; bli = li;",
                         "          if (r.status == FO_CAND_OK && r.makespan <= bft) {\n            if (bg) { fo_graph_free(bg); fo_result_free(&br); }\n            bg = sv; br = r; bft = r.makespan; bli = li;", None),
    "live_never_frees": ("R24", "if (--rem[m] == 0) used[r->place[m]] -= g->mem[m] - g->param[m];",
                         "if (--rem[m] == 0) used[r->place[m]] -= 0;", None),
}


def apply(src, old, new, occ):
    n = src.count(old)
    if occ is None:
        assert n == 1, "mutation anchor must be unique (found %d): %r" % (n, old)
        return src.replace(old, new)
    assert n > occ, "anchor %r found %d times" % (old, n)
    pos = -1
    for _ in range(occ + 1):
        pos = src.index(old, pos + 1)
    return src[:pos] + new + src[pos + len(old):]


def main(names):
    base = open(SRC).read()
    rows = []
    for name in names or list(MUTANTS):
        cite, old, new, occ = MUTANTS[name]
        path = "/tmp/mut_%s.c" % name
        with open(path, "w") as f:
            f.write(apply(base, old, new, occ))
        env = dict(os.environ, FASTT_ORACLE_SRC=path)
        t = time.time()
        p = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider"] + PINS, cwd=ROOT,
                           env=env, capture_output=True, text=True)
        first = next((l for l in p.stdout.splitlines() if l.startswith("FAILED")), "")
        rows.append((name, cite, p.returncode != 0, first.replace("FAILED ", "")[:90], time.time() - t))
        print("%-30s %-22s %-8s %s" % (name, cite, "killed" if rows[-1][2] else "SURVIVED", rows[-1][3]), flush=True)
    return 0 if all(r[2] for r in rows) else 1


if __name__ == "__main__":
    sys.exit(main(sys.argv[1:]))
