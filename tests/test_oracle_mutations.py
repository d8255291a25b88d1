"""Mutation check of the oracle's pins (CPU only).

Every GPU parity claim rests on oracle/oracle.cpp, so its pins must catch plausible
mistakes.  Each case below copies the oracle, the shared input generators and the oracle
pin tests into a scratch directory, applies one plausible mistake to oracle.cpp (a
dropped term, a flipped rule, a swapped draw order, a wrong scale, a transposed
operand), rebuilds it and runs the pin suite there: the named pin test must fail.
The product library is never involved.
"""
import os
import shutil
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PIN_FILES = ["tests/test_oracle_plan.py", "tests/test_oracle_lsh.py", "tests/test_oracle_numeric.py"]

# (name, original snippet, mutated snippet, a pin test that must fail)
MUTATIONS = [
    ("auto_round2_inverted",  # P:332 "skip round 2 if AvgSim > 0.1" inverted
     "round2 = !((unsigned __int128)snum * d2 > (unsigned __int128)n2 * sden);",
     "round2 = ((unsigned __int128)snum * d2 > (unsigned __int128)n2 * sden);",
     "test_auto_skips_round2_when_remainder_is_clustered"),
    ("auto_round2_not_strict",  # "greater than" read as >=
     "round2 = !((unsigned __int128)snum * d2 > (unsigned __int128)n2 * sden);",
     "round2 = !((unsigned __int128)snum * d2 >= (unsigned __int128)n2 * sden);",
     "test_auto_round2_threshold_is_strict"),
    ("auto_round1_inverted",  # P:332 "skip round 1 if DenseRatio > 10%" inverted
     "if (mode == 0) round1 = !((unsigned __int128)dense0 * d1 > (unsigned __int128)n1 * nnz);",
     "if (mode == 0) round1 = ((unsigned __int128)dense0 * d1 > (unsigned __int128)n1 * nnz);",
     "test_auto_skips_round1_on_clustered_matrix"),
    ("auto_threshold_ignored",  # R28: the decision's own dense criterion
     "const int32_t dense_min0 = auto_dense_min > 0 ? auto_dense_min : dense_min;",
     "const int32_t dense_min0 = dense_min;",
     "test_auto_decision_threshold_separate_from_execution_threshold"),
    ("sddmm_bound_scale_x100",  # tolerance scale of every GPU SDDMM check
     "if (out_abs) out_abs[j] = accabs * std::abs((double)vals[j]);",
     "if (out_abs) out_abs[j] = 100.0 * accabs * std::abs((double)vals[j]);",
     "test_sddmm_bound_scale_elementwise"),
    ("hash_draw_order_swapped",  # R13: a_s drawn before b_s
     "    a[s] = (uint32_t)(splitmix64_next(&state) & 0xFFFFFFFFull) | 1u;\n"
     "    b[s] = (uint32_t)(splitmix64_next(&state) & 0xFFFFFFFFull);",
     "    b[s] = (uint32_t)(splitmix64_next(&state) & 0xFFFFFFFFull);\n"
     "    a[s] = (uint32_t)(splitmix64_next(&state) & 0xFFFFFFFFull) | 1u;",
     "test_hash_params_draw_order"),
    ("sddmm_missing_value_factor",  # Alg 2 line "O.value[j] *= S.value[j]" dropped
     "out[j] = acc * (double)vals[j];",
     "out[j] = acc;",
     "test_sddmm_matches_dense_bruteforce"),
    ("spmm_reversed_k",  # B row read back to front (a transposed / mis-indexed operand)
     "for (int64_t k = 0; k < K; ++k) c[k] += (double)vals[j] * (double)x[k];",
     "for (int64_t k = 0; k < K; ++k) c[k] += (double)vals[j] * (double)x[K - 1 - k];",
     "test_spmm_matches_dense_bruteforce"),
    ("tie_goes_to_larger_index",  # R6: equal size -> smaller index wins
     "if (cluster_sz[i] > cluster_sz[j] || (cluster_sz[i] == cluster_sz[j] && i < j)) {",
     "if (cluster_sz[i] > cluster_sz[j] || (cluster_sz[i] == cluster_sz[j] && i > j)) {",
     "test_equal_size_root_is_smaller_index_output_order"),
    ("size_update_dropped",  # R4: sz[winner] += sz[loser]
     "      cluster_sz[w] += cluster_sz[l];\n",
     "",
     "test_size_update_drives_threshold_deletion"),
    ("tiler_column_order_ascending_count",  # R18: (count desc, column asc)
     "if (cnt[x] != cnt[y]) return cnt[x] > cnt[y];",
     "if (cnt[x] != cnt[y]) return cnt[x] < cnt[y];",
     "test_aspt_after_reordering_fig4"),
]


def _scratch(tmp_path):
    for d in ("oracle", "synth", "tests"):
        shutil.copytree(os.path.join(ROOT, d), tmp_path / d,
                        ignore=shutil.ignore_patterns("*.so", "__pycache__", "*.tmp"))
    shutil.copy(os.path.join(ROOT, "pytest.ini"), tmp_path / "pytest.ini")
    return tmp_path


@pytest.mark.parametrize("name,orig,mut,test", MUTATIONS, ids=[m[0] for m in MUTATIONS])
def test_mutation_is_caught(tmp_path, name, orig, mut, test):
    d = _scratch(tmp_path)
    src = d / "oracle" / "oracle.cpp"
    text = src.read_text()
    assert text.count(orig) == 1, f"mutation site of {name} not found exactly once"
    src.write_text(text.replace(orig, mut))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider", "-k", test] + PIN_FILES,
                       cwd=d, capture_output=True, text=True, timeout=600)
    assert r.returncode == 1 and " failed" in r.stdout, \
        f"mutation {name} survived the pins:\n{r.stdout[-2000:]}\n{r.stderr[-2000:]}"
