# per-thread link masks in the CTA water-filling: parity (incl. C5 goldens <= 256 GPUs), phase profile, C5 group times
O=gpurun_out/s4l
mkdir -p $O
timeout 1800 python -m pytest tests -m gpu -q -x > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRIOSIM_LIB=paper_conf_isca_libwmvgjbj025_b200/libtriosim_prof.so timeout 600 python tools/c5_prof.py 64 512 1024 > $O/c5prof.log 2>&1
timeout 900 python tools/c5_subset.py 64 128 256 > $O/c5sub.log 2>&1; echo "rc=$?" >> $O/c5sub.log
ls -la $O
