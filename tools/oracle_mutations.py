"""Mutation check of the oracle decoder: delete one rejection branch of
oracle_decompress at a time (in a copy of the repo under /tmp) and run the
oracle pins; every mutation must fail at least one pin.

    python tools/oracle_mutations.py
"""
import os, shutil, subprocess
muts = [
 ("d > W", "if (d > W || d > produced || L > F || L > m - produced)", "if (d > produced || L > F || L > m - produced)"),
 ("L > F", "if (d > W || d > produced || L > F || L > m - produced)", "if (d > W || d > produced || L > m - produced)"),
 ("version", "if (get_le(in + 4, 2) != 1 || get_le(in + 6, 2) != OR_HEADER_BYTES)", "if (get_le(in + 6, 2) != OR_HEADER_BYTES)"),
 ("header_bytes", "if (get_le(in + 4, 2) != 1 || get_le(in + 6, 2) != OR_HEADER_BYTES)", "if (get_le(in + 4, 2) != 1)"),
 ("C", "if (C != n_chunks(n, S)) return OR_ERR_CORRUPT;", ""),
]
for name, a, b in muts:
    r = "/tmp/mut/r"
    shutil.rmtree(r, ignore_errors=True)
    os.makedirs(r)
    for d in ("oracle", "tests", "paper_conf_cluster_ozsoys11_b200"):
        shutil.copytree("/root/repo/" + d, f"{r}/{d}", ignore=shutil.ignore_patterns("*.so"))
    shutil.copy("/root/repo/pytest.ini", r)
    src = open(f"{r}/oracle/culzss_oracle.c").read()
    assert a in src, name
    open(f"{r}/oracle/culzss_oracle.c", "w").write(src.replace(a, b))
    out = subprocess.run("python -m pytest tests/test_oracle_pins.py tests/test_oracle_bruteforce.py -q -m 'not gpu' 2>&1 | tail -3",
                         shell=True, cwd=r, capture_output=True, text=True).stdout
    print(name, "->", out.strip().splitlines()[-1])
