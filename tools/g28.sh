for v in 0 1; do DT_HOST_PIPE=$v python tools/host_probe.py; done
DT_HOST_CHUNK=16777216 python tools/host_probe.py
DT_HOST_CHUNK=2097152 python tools/host_probe.py
