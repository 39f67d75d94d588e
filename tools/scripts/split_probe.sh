for f in 256 512 768 1024; do python tools/block_probe.py C2A $f; done
for f in 256 512 768; do python tools/block_probe.py C2B $f; done
for f in 0 256 512; do python tools/block_probe.py C3 $f; done
