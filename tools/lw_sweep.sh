# knob sweep on the pipelined concurrent-stream step: VAR, VALUES
for v in $VALUES; do echo "== $VAR $v"; export $VAR=$v
KS=${KS:-2,3} timeout 300 python tools/instances.py 2>&1 | grep "pipelined=True"
done
