"""Ranked report / folded-function grouping (S8(f) #1)."""
import json

import numpy as np
import pytest

from paper_conf_sc_weltonm19_b200 import report


def test_demangle_and_fold_names():
    assert report.demangle("_ZN3als4stepEv") == "als::step()"
    assert report.fold_function_name("_ZN6thrust6detail3fooIiEEvPi") == "thrust::detail::foo"
    # template instances that differ only by parameter types fold together
    a = report.fold_function_name("void cusp::multiply<float, int>(cusp::csr_matrix<int,float> const&)")
    b = report.fold_function_name("void cusp::multiply<double, long>(cusp::csr_matrix<long,double> const&)")
    assert a == b == "cusp::multiply"
    assert report.fold_function_name("std::vector<int, std::allocator<int> >::push_back(int const&)") == \
        "std::vector::push_back"
    assert report.fold_function_name("cudaMemcpy") == "cudaMemcpy"
    assert report.fold_function_name("bool operator<(A const&, B const&)") == "operator<"
    assert report.fold_function_name("foo(int) const") == "foo"


def test_group_sites():
    g, names = report.group_sites(["f<int>(int)", "g()", "f<float>(float)", "_ZN3als4stepEv"])
    assert g.tolist() == [0, 1, 0, 2] and names == ["f", "g", "als::step"]


def test_ranked_report_orders_and_totals():
    ben = np.array([5, 0, 30, 10], np.uint64)
    cnt = np.array([1, 0, 3, 2], np.uint64)
    names = ["als.cpp:738", "als.cpp:739", "als.cpp:760", "x.cu:1"]
    funcs = ["f<int>()", "g()", "f<long>()", "h()"]
    with pytest.raises(ValueError):          # the group sums are the device's (ffm_fold_sites)
        report.ranked_report(ben, names, cnt, funcs)

    def fold(v, g, n):                       # stands in for FfmLog.fold on a CPU-only box
        out = np.zeros(n, np.uint64)
        np.add.at(out, np.asarray(g, np.int64), np.asarray(v, np.uint64))
        return out
    rep = report.ranked_report(ben, names, cnt, funcs, fold=fold, exec_time_ns=100)
    assert [r["name"] for r in rep["single_point"]] == ["als.cpp:760", "x.cu:1", "als.cpp:738"]
    assert rep["total"] == {"benefit_ns": 45, "benefit_s": 45e-9, "transfer_issues": 3, "pct_exec": 45.0,
                            "duplicates": 6}
    assert [(r["name"], r["benefit_ns"]) for r in rep["folded_function"]] == [("f", 35), ("h", 10)]
    assert json.loads(report.to_json(rep))["single_point"][0]["pct_exec"] == 30.0
