"""The driver's round-end smoke(): one small config-1-shaped log on cuda:0 through the C ABI,
checked element by element against the oracle (duplicate_of, benefit_ns)."""
import pytest

import __graft_entry__


@pytest.mark.gpu
def test_smoke_entry(capsys):
    __graft_entry__.smoke()
    assert "smoke ok" in capsys.readouterr().out
