"""scripts/nvlink_summary.py (the multi-GPU NVLink / PCIe counter summary behind bench.py's
N > 1 roofline.traffic) on CSVs shaped like `ncu --csv` output, with template kernel
names: per-kernel GB/s from the summed bytes over the summed kernel time, and the key
bench.py reads."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = ('"ID","Process ID","Process Name","Host Name","Kernel Name","Context","Stream","Block Size",'
       '"Grid Size","Device","CC","Section Name","Metric Name","Metric Unit","Metric Value"\n')


def row(i, kernel, metric, unit, value):
    return (f'"{i}","1","python3","127.0.0.1","{kernel}","1","13","(256, 1, 1)","(296, 1, 1)","0","10.0",'
            f'"Command line profiler metrics","{metric}","{unit}","{value}"\n')


def test_summary_keys_and_rates(tmp_path):
    send = "void mpx::<unnamed>::send_kernel<6>(mpx::SendParams)"
    relay = "void mpx::<unnamed>::relay_kernel<4>(mpx::RelayParams)"
    with open(tmp_path / "ncu_rank0.csv", "w") as f:
        f.write("==PROF== Connected\n" + HDR)
        for i in range(2):  # two launches of 1 ms each moving 0.5 GB over NVLink
            f.write(row(3 * i, send, "gpu__time_duration.sum", "ns", "1,000,000"))
            f.write(row(3 * i + 1, send, "nvltx__bytes_data_user.sum", "byte", "500,000,000"))
            f.write(row(3 * i + 2, send, "pcie__write_bytes.sum", "byte", "32000000"))
    with open(tmp_path / "ncu_rank2.csv", "w") as f:
        f.write(HDR + row(0, relay, "gpu__time_duration.sum", "ns", "2000000")
                + row(1, relay, "nvlrx__bytes_data_user.sum", "byte", "300000000"))
    out = tmp_path / "nvl.json"
    subprocess.run([sys.executable, os.path.join(ROOT, "scripts", "nvlink_summary.py"), str(tmp_path), "3",
                    str(1 << 30), "--out", str(out)], check=True, capture_output=True, text=True)
    doc = json.load(open(out))[f"3:{1 << 30}"]
    s = doc["rank0:send_kernel"]          # the key bench.py's N > 1 line reads
    assert s["launches"] == 2 and abs(s["avg_us"] - 1000.0) < 1e-6
    assert abs(s["nvlink_tx_GBps"] - 500.0) < 1e-9 and abs(s["frac_tx_of_900"] - 500.0 / 900.0) < 1e-12
    assert abs(s["pcie_write_GBps"] - 32.0) < 1e-9 and s["nvlink_tx_bytes_per_launch"] == 5e8
    r = doc["rank2:relay_kernel"]
    assert abs(r["nvlink_rx_GBps"] - 150.0) < 1e-9 and r["nvlink_tx_GBps"] == 0.0
