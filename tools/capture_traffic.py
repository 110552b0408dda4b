"""Write profiles/decode_traffic.json from an `ncu --set full` capture of ONE
decode launch, stamped with the hash of the decode kernel source, so bench.py
reports roofline.traffic only for the kernel that was actually profiled.

    ncu --set full --clock-control none -k regex:decode_kernel -s 2 -c 1 \\
        -o gpurun_out/decode_traffic python tools/prof_decode.py --sms 4 --tasks 3
    python tools/capture_traffic.py gpurun_out/decode_traffic.ncu-rep
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from workloads.configs import GPT2S  # noqa: E402


def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    def metric(name):
        i = hdr.index(name)
        v = float(vals[i].replace(",", ""))
        u = units[i]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        return v * scale
    rd, wr = metric("dram__bytes_read.sum"), metric("dram__bytes_write.sum")
    d = {"kernel": "decode_kernel<1> (GPT-2s task, 4-SM partition)",
         "dram_bytes_per_launch": int(rd + wr), "dram_read_bytes": int(rd),
         "dram_write_bytes": int(wr),
         "algorithmic_bytes_per_launch": bench.task_bytes(GPT2S, 1, bench.P_LEN, bench.G_LEN),
         "source": f"ncu --set full ({os.path.basename(rep)})",
         "source_sha256": bench.kernel_source_hash()}
    with open(os.path.join(ROOT, "profiles", "decode_traffic.json"), "w") as f:
        json.dump(d, f, indent=1)
    print(json.dumps(d))


if __name__ == "__main__":
    main(sys.argv[1])
