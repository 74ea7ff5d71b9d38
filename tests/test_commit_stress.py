"""The library's commit engine under real concurrency, compiled with ThreadSanitizer (SURVEY §4:
"free-queue / CAS stress under -fsanitize=thread").  N+1 writer threads per rank race through
Listing 1 — begin / FILLING / complete — while a checker thread asserts the
L229 invariants and, for W = 2, runs the R20 commit rule (MIN of the local latest, apply_global)
and asserts every rank still holds g.  Afterwards the oracle, which shares no code with the
engine, must restore exactly the iter the engine reports from the files it left."""
import os
import subprocess

import numpy as np
import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CSRC = os.path.join(ROOT, "paper_conf_asplos_strati0k25_b200", "csrc")
CB, CHUNKS = 4096, 6


def _build(tmp_path_factory, san):
    out = os.path.join(ROOT, "build", f"commit_stress_{san}")
    srcs = [os.path.join(ROOT, "tests", "native", "commit_stress.cpp"), os.path.join(CSRC, "commit.cpp"),
            os.path.join(CSRC, "host_api.cpp")]
    newest = max(os.path.getmtime(p) for p in srcs + [os.path.join(CSRC, f) for f in os.listdir(CSRC)])
    if not os.path.exists(out) or os.path.getmtime(out) < newest:
        os.makedirs(os.path.dirname(out), exist_ok=True)
        flag = {"tsan": "-fsanitize=thread", "asan": "-fsanitize=address,undefined -fno-sanitize-recover=all"}[san]
        subprocess.run(["g++", "-std=c++17", "-O1", "-g", "-msse4.2", *flag.split(), "-I/usr/local/cuda/include",
                        "-o", out, *srcs, "-lpthread"], check=True, capture_output=True, text=True)
    return out


@pytest.fixture(scope="module", params=["tsan", "asan"])
def stress_bin(request, tmp_path_factory):
    return request.param, _build(tmp_path_factory, request.param)


@pytest.mark.parametrize("N,world,seed", [(1, 1, 1), (2, 1, 2), (3, 1, 3), (2, 2, 4), (1, 2, 5)])
def test_commit_engine_concurrent_invariants(stress_bin, tmp_path, N, world, seed):
    san, exe = stress_bin
    lcrc = oracle.layout_crc([CB * CHUNKS], [0], 256, CB)
    env = dict(os.environ, TSAN_OPTIONS="halt_on_error=1 exitcode=66", ASAN_OPTIONS="detect_leaks=1")
    r = subprocess.run([exe, str(tmp_path), str(N), str(world), "300", str(seed), str(lcrc)], capture_output=True,
                       text=True, timeout=300, env=env)
    assert r.returncode == 0, f"{san}: rc={r.returncode}\n{r.stdout}\n{r.stderr[-4000:]}"
    assert "WARNING: ThreadSanitizer" not in r.stderr, r.stderr[-4000:]
    line = r.stdout.strip().splitlines()[-1].split()
    assert line[0] == "OK", r.stdout
    latest0, g = int(line[1]), int(line[2])
    paths = [str(tmp_path / f"rank{k}.pcc") for k in range(world)]
    rc, it, bad, outs = oracle.restore(paths, N + 1, [CB * CHUNKS], [0], 256, CB)
    assert rc == 0 and not bad, (rc, bad)
    # W = 1: the newest committed checkpoint; W > 1: the last global id every rank agreed on
    assert it == (latest0 if world == 1 else g)
    assert not outs[0].any()  # the writers never wrote data: the sparse slots read back as zeros
