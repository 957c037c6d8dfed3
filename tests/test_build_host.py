"""Host logic of the build: the instantiation units generated from csrc/instantiations.txt and
the path-independent content hash (no GPU needed)."""
import os

from paper_conf_ipps_juryl022_b200 import build


def test_generated_units_match_the_spec(tmp_path):
    paths = build.generate_units(str(tmp_path))
    spec = [ln for ln in open(build.SPEC) if ln.strip() and not ln.startswith("#")]
    assert len(paths) == len(spec) == len(set(paths))
    for p, ln in zip(paths, spec):
        name, header, guard, insts = [x.strip() for x in ln.split("|", 3)]
        src = open(p).read()
        assert os.path.basename(p) == f"inst_{name}.cu"
        assert f'#include "{header}"' in src and "#define MP_DIAG_IMPL" in src
        assert src.count("template struct ") == len([x for x in insts.split(";") if x.strip()])
        assert (f"#if {guard}" in src) == (guard != "-")
        assert os.path.exists(os.path.join(build.CSRC, header))


def test_generation_is_idempotent(tmp_path):
    build.generate_units(str(tmp_path))
    stamps = {p: os.stat(p).st_mtime_ns for p in build.generate_units(str(tmp_path))}
    again = build.generate_units(str(tmp_path))
    assert {p: os.stat(p).st_mtime_ns for p in again} == stamps   # unchanged files are not rewritten


def test_digest_is_path_independent():
    cmd = " ".join([build.NVCC] + build.ARCH + build.FLAGS)
    assert build.HERE not in build._rel(cmd) and "<pkg>" in build._rel(cmd)
