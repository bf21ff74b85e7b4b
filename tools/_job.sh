bash tools/gpu.sh h12 build smoke suite bench
for c in amazoncat13k wiki10_31k amazon670k; do bash tools/gpu.sh h12 bench:$c; done
