"""Command-line front end (python -m paper_conf_sosp_kamathb21_b200): argument parsing, trace-file
reading and CSV writing on CPU; the full run (GPU) against the oracle."""
import io
import os
import subprocess
import sys

import numpy as np
import pytest

import tracegen as tg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_parse_and_read(tmp_path):
    from paper_conf_sosp_kamathb21_b200 import __main__ as cli

    ev, nb, bd = tg.random_trace(7, 50)
    p = tmp_path / "t.bin"
    ev.tofile(p)
    a = cli.parse_args([str(p), "--blocks", str(nb), "--block-dim", str(bd), "--coalesce"])
    assert a.blocks == nb and a.block_dim == bd and a.coalesce and not a.paper_counters
    back = cli.read_trace(str(p))
    assert np.array_equal(back.view(np.uint8), ev.view(np.uint8))


def test_rejects_partial_record(tmp_path):
    from paper_conf_sosp_kamathb21_b200 import __main__ as cli

    p = tmp_path / "bad.bin"
    p.write_bytes(b"\0" * 17)
    with pytest.raises(SystemExit):
        cli.read_trace(str(p))


def test_csv_format():
    from paper_conf_sosp_kamathb21_b200 import __main__ as cli

    r = np.zeros(2, tg.REPORT_DTYPE)
    r["addr"] = [0x40, 0x80]
    r["cur"] = [5, 9]
    r["prev"] = [1, 2]
    r["type"] = [4, 2]
    buf = io.StringIO()
    cli.write_csv(r, buf)
    assert buf.getvalue().splitlines() == ["addr,cur,prev,type,cur_kind,prev_kind", "0x40,5,1,4,0,0", "0x80,9,2,2,0,0"]


@pytest.mark.gpu
def test_cli_matches_oracle(tmp_path):
    import oracle
    import tracegen.families as F

    ev, nb, bd, _ = F.generate(1)
    p = tmp_path / "c1.bin"
    ev.tofile(p)
    out = tmp_path / "r.csv"
    subprocess.run([sys.executable, "-m", "paper_conf_sosp_kamathb21_b200", str(p), "--blocks", str(nb),
                    "--block-dim", str(bd), "--out", str(out)], cwd=ROOT, check=True, capture_output=True)
    rows = out.read_text().splitlines()[1:]
    want = oracle.run(ev, nb, bd)
    assert [tuple(int(x, 0) for x in row.split(",")) for row in rows] == \
           [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"]), int(r["cur_kind"]), int(r["prev_kind"]))
            for r in want]
