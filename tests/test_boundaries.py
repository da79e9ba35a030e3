"""Separation rules, checked on the sources (CPU): the product package never
imports or links anything under oracle/; the oracle never uses the product;
synth/ (the seeded inputs both sides share) holds neither side; the CUDA
sources include no oracle header.  bench.py touches oracle/ only in its
cpu_baseline / reference legs."""
import ast
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_icpp_yecrbypnmskn24_b200")


def py_imports(path):
    tree = ast.parse(open(path).read())
    mods = set()
    for node in ast.walk(tree):
        if isinstance(node, ast.Import):
            mods |= {a.name.split(".")[0] for a in node.names}
        elif isinstance(node, ast.ImportFrom) and node.module:
            mods.add(node.module.split(".")[0])
    return mods


def files(d, exts):
    for dp, _, fs in os.walk(d):
        if "__pycache__" in dp or "/build" in dp:
            continue
        for f in fs:
            if f.endswith(exts):
                yield os.path.join(dp, f)


def test_product_package_never_imports_the_oracle():
    for f in files(PKG, (".py",)):
        assert "oracle" not in py_imports(f), f


def test_cuda_sources_include_no_oracle_code():
    for f in files(os.path.join(PKG, "csrc"), (".cu", ".cpp", ".h", ".c")):
        src = open(f).read()
        assert not re.search(r'#include\s+[<"][^>"]*oracle', src), f


def test_oracle_never_uses_the_product():
    for f in files(os.path.join(ROOT, "oracle"), (".py",)):
        assert not {"paper_conf_icpp_yecrbypnmskn24_b200", "synth"} & py_imports(f) - {"synth"}, f
    src = open(os.path.join(ROOT, "oracle", "viper_oracle.c")).read()
    assert not re.search(r'#include\s+[<"][^>"]*(csrc|viper\.h|vp_internal|runtime\.h)', src)


def test_shared_inputs_hold_neither_side():
    for f in files(os.path.join(ROOT, "synth"), (".py",)):
        assert not {"oracle", "paper_conf_icpp_yecrbypnmskn24_b200"} & py_imports(f), f


def test_bench_uses_the_oracle_only_in_its_baseline_legs():
    """Only the OracleUpdates helper imports oracle/, and only the
    cpu_baseline and reference legs construct it."""
    tree = ast.parse(open(os.path.join(ROOT, "bench.py")).read())
    top = {n.module for n in tree.body if isinstance(n, ast.ImportFrom) and n.module}
    top |= {a.name for n in tree.body if isinstance(n, ast.Import) for a in n.names}
    assert not any(m.startswith("oracle") for m in top)
    importers, users, par_users = set(), set(), set()
    scopes = [n for n in ast.walk(tree) if isinstance(n, (ast.FunctionDef, ast.ClassDef))]
    for sc in scopes:
        for node in ast.walk(sc):
            if isinstance(node, ast.ImportFrom) and node.module and node.module.startswith("oracle"):
                importers.add(sc.name)
            if isinstance(node, ast.Import) and any(a.name.startswith("oracle") for a in node.names):
                importers.add(sc.name)
            if isinstance(sc, ast.FunctionDef) and isinstance(node, ast.Call) and \
                    getattr(node.func, "id", None) == "OracleUpdates":
                users.add(sc.name)
            if isinstance(sc, ast.FunctionDef) and isinstance(node, ast.Call) and \
                    getattr(node.func, "id", None) == "oracle_parallel":
                par_users.add(sc.name)
    assert importers <= {"OracleUpdates", "__init__"} and "OracleUpdates" in importers, importers
    # oracle_parallel (the P-thread oracle baseline) is part of the cpu_baseline leg only
    assert users and users <= {"cpu_baseline", "reference_arm", "oracle_parallel"}, users
    assert par_users <= {"cpu_baseline"}, par_users
