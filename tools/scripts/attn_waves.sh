for f in 0 16 32; do
python tools/attn_probe.py 1229 4096 10 64 4 $f
python tools/attn_probe.py 307 1024 20 64 4 $f
python tools/attn_probe.py 4096 4096 10 64 4 $f
python tools/attn_probe.py 1331 4608 24 128 1 $f
python tools/attn_probe.py 1843 4608 24 128 16 $f
done
