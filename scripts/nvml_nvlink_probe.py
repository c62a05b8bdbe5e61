"""Which NVML NVLink counters this driver/GPU supports (run on the GPU box): link states, and the
return code + value of the data-byte fields bench.py's NvLink class reads (202/204 bytes,
138/139 KiB), per active link.  One line of JSON."""
import json

import pynvml

pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
links = []
for l in range(18):
    try:
        if pynvml.nvmlDeviceGetNvLinkState(h, l) == 1:
            links.append(l)
    except Exception as e:
        links.append(f"err {e}")
        break
out = {"driver": pynvml.nvmlSystemGetDriverVersion(), "links_active": links, "fields": {}}
for f in (202, 204, 138, 139, 140, 141):
    res = []
    for l in [x for x in links if isinstance(x, int)][:3]:
        v = pynvml.nvmlDeviceGetFieldValues(h, [(f, l)])[0]
        res.append({"link": l, "ret": v.nvmlReturn, "value": int(v.value.ullVal) if v.nvmlReturn == 0 else None})
    out["fields"][f] = res
print(json.dumps(out))
