"""Independent pin of the semantic programs' expected values
(orc_sem_expected, SURVEY PIN-13): the same programs written as ordinary host
OpenMP (tests/omp_host/sem_omp.c) and executed by gcc's libgomp -- a real
OpenMP implementation decides every level, team size, ancestor thread number,
ICV and static-chunk owner, instead of a restated formula."""
import os
import shutil
import subprocess

import numpy as np
import pytest

HERE = os.path.dirname(os.path.abspath(__file__))


@pytest.fixture(scope="module")
def sem_omp(tmp_path_factory):
    if shutil.which("gcc") is None:
        pytest.skip("gcc not available")
    exe = str(tmp_path_factory.mktemp("omp") / "sem_omp")
    subprocess.check_call(["gcc", "-O1", "-fopenmp", os.path.join(HERE, "omp_host", "sem_omp.c"), "-o", exe])
    return exe


def _run(exe, test, G, T):
    r = subprocess.run([exe, str(test), str(G), str(T)], capture_output=True, text=True, check=True,
                       env=dict(os.environ, OMP_THREAD_LIMIT="4096"), timeout=120)
    return np.array([int(x) for x in r.stdout.split()], dtype=np.uint64)


@pytest.mark.parametrize("G,T", [(5, 64), (3, 32), (2, 128), (4, 96)])
@pytest.mark.parametrize("test", range(9))
def test_semantics_equal_libgomp(orc, sem_omp, test, G, T):
    want = _run(sem_omp, test, G, T)
    got = orc.sem_expected(test, G, T)
    assert len(got) == len(want)
    assert np.array_equal(got, want), (test, np.nonzero(got != want)[0][:8])
